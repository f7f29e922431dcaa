#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02e_build.log 2>&1
bash tools/prof.sh full r02e_screen k_screen_f16
bash tools/prof.sh list r02e_c4

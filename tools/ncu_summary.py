"""Summarise an ncu raw CSV page (ncu -i X.ncu-rep --page raw --csv)."""
import csv
import sys

KEYS = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 'lts__t_sector_hit_rate.pct',
        'sm__throughput.avg.pct_of_peak_sustained_elapsed', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'launch__registers_per_thread', 'sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active',
        'l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum', 'smsp__inst_executed.sum',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'launch__grid_size', 'launch__block_size',
        'sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum']
# prefixes printed for every matching counter (tensor pipe, L2 throughput)
PREFIXES = ['sm__pipe_tensor', 'sm__pipe_tc', 'sm__inst_executed_pipe_tc', 'lts__t_bytes.sum',
            'lts__throughput.avg.pct', 'l1tex__throughput.avg.pct', 'sm__pipe_shared_cycles_active']


def main(path, top=12):
    r = list(csv.reader(open(path)))
    hdr, units, vals = r[0], r[1], r[2]
    for w in KEYS:
        for i, h in enumerate(hdr):
            if h == w:
                print(f"{w:70s} {vals[i]:>20s} {units[i]}")
    for i, h in enumerate(hdr):
        if any(h.startswith(p) for p in PREFIXES):
            print(f"{h:70s} {vals[i]:>20s} {units[i]}")
    st = []
    for i, h in enumerate(hdr):
        if h.startswith('smsp__pcsamp_warps_issue_stalled') and not h.endswith('not_issued'):
            try:
                st.append((float(vals[i].replace(',', '')), h.replace('smsp__pcsamp_warps_issue_stalled_', '')))
            except ValueError:
                pass
    tot = sum(v for v, _ in st) or 1
    print("stall samples:", ", ".join(f"{h} {100*v/tot:.0f}%" for v, h in sorted(st, reverse=True)[:top]))


if __name__ == "__main__":
    main(sys.argv[1])

"""Aggregate ncu per-instruction stall samples by CUDA source line.

    python tools/ncu_lines.py <rep.ncu-rep | source-page.csv> <kernel-substring> [top]

Reads the SASS source page of the capture (`ncu -i … --page source --csv`), maps
each instruction offset to its source line with `nvdisasm -g` of the kernel's
cubin in the in-tree library (must be the library the capture ran), and prints
the lines with the most warp-stall samples.
"""
import collections
import csv
import io
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.environ.get("BLSH_LIB") or os.path.join(ROOT, "paper_conf_icde_panm12_b200", "_lib", "libblsh.so")


def line_map(kernel_sub):
    tmp = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", LIB], cwd=tmp, capture_output=True, check=True)
    for f in sorted(os.listdir(tmp)):
        out = subprocess.run(["nvdisasm", "-g", os.path.join(tmp, f)], capture_output=True, text=True).stdout
        m = None
        for sec in re.split(r"\n\s*\.section\s+", out):
            if sec.startswith(".text.") and kernel_sub in sec.split("\n", 1)[0]:
                m = sec
                break
        if m is None:
            continue
        res, loc = {}, "?"
        for ln in m.splitlines():
            if "//## File" in ln:
                g = re.search(r'File "([^"]+)", line (\d+)', ln)
                loc = f"{os.path.basename(g.group(1))}:{g.group(2)}" if g else "?"
            g = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", ln)
            if g:
                res[int(g.group(1), 16)] = (loc, g.group(2).strip())
        return res
    raise SystemExit(f"kernel {kernel_sub} not found in {LIB}")


def main():
    rep, ksub = sys.argv[1], sys.argv[2]
    top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
    if rep.endswith(".csv"):   # an exported source page (ncu -i rep --page source --csv > file.csv)
        txt = open(rep).read()
    else:
        txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr = rows[1]
    ia, isamp, iex = hdr.index("Address"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
    body = [r for r in rows[2:] if len(r) > isamp and r[ia].startswith("0x")]
    base = int(body[0][ia], 16)
    lm = line_map(ksub)
    agg = collections.Counter()
    ex = collections.Counter()
    stalls = [(i, h) for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
    why = collections.defaultdict(collections.Counter)
    tot = 0
    for r in body:
        off = int(r[ia], 16) - base
        loc = lm.get(off, ("?", ""))[0]
        s = int(r[isamp] or 0)
        agg[loc] += s
        ex[loc] += int(r[iex] or 0)
        for i, h in stalls:
            try:
                why[loc][h[6:]] += int(r[i] or 0)
            except ValueError:
                pass
        tot += s
    print(f"total samples {tot}")
    for loc, s in agg.most_common(top):
        w = ", ".join(f"{k} {v * 100 // max(s, 1)}%" for k, v in why[loc].most_common(2) if v)
        print(f"{100.0 * s / max(tot, 1):6.2f}%  {s:9d}  inst {ex[loc]:12d}  {loc}  [{w}]")


if __name__ == "__main__":
    main()

"""Aggregate ncu SASS-level warp-stall samples onto CUDA source lines
(nvdisasm -g line table of the cubin extracted from libnorthup.so)."""
import csv, re, subprocess, sys, os, tempfile, glob
from collections import Counter
rep, cu = sys.argv[1], sys.argv[2]          # report, source file basename (leaf_2sm)
lib = sys.argv[3] if len(sys.argv) > 3 else "paper_conf_ipps_chey19_b200/libnorthup.so"
func = sys.argv[4] if len(sys.argv) > 4 else None
d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(lib)], cwd=d, capture_output=True)
cub = glob.glob(os.path.join(d, f"{cu}.sm_100a.cubin"))[0]
sass = subprocess.run(["nvdisasm", "-g", "-c", cub], capture_output=True, text=True).stdout.split("\n")
cur = None; off2line = {}
for l in sass:
    m = re.search(r'//## File ".*?", line (\d+)', l)
    if m: cur = int(m.group(1)); continue
    m = re.match(r'\s*/\*([0-9a-f]{4,})\*/', l)
    if m and cur is not None: off2line[int(m.group(1), 16)] = cur
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = rows[1]; ia = hdr.index("Address"); iw = hdr.index("Warp Stall Sampling (All Samples)")
base = int(rows[2][ia], 16)
src = open(glob.glob(f"paper_conf_ipps_chey19_b200/csrc/{cu}.cu")[0]).read().split("\n")
agg = Counter(); tot = 0
for r in rows[2:]:
    try: a = int(r[ia], 16) - base; w = int(r[iw] or 0)
    except Exception: continue
    tot += w; agg[off2line.get(a, -1)] += w
print("total samples", tot)
for ln, w in agg.most_common(int(os.environ.get("TOP", "25"))):
    print(f"{w:8d} {100*w/tot:5.1f}%  L{ln:4d}  {src[ln-1].strip()[:90] if ln > 0 else '?'}")

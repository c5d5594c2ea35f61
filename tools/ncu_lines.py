"""Attribute an ncu SASS source page (k_main, --page source --csv --print-source sass)
to CUDA source lines with the line table of the same librcm.so (nvdisasm).
usage: python tools/ncu_lines.py <sass.csv> <all.sass> [kernel-prefix]"""
import collections, csv, re, sys
sass_csv, dis = sys.argv[1], sys.argv[2]
kname = sys.argv[3] if len(sys.argv) > 3 else ".text._Z6k_mainILi2"
lines = open(dis).read().splitlines()
start = [i for i, l in enumerate(lines) if l.startswith(kname)][0]
amap, cur = {}, None
for l in lines[start + 1:]:
    if l.startswith(".text._Z"):
        break
    m2 = re.search(r'//## File "([^"]+)", line (\d+)', l)
    if m2:
        cur = (m2.group(1).split("/")[-1], int(m2.group(2)))
    m3 = re.search(r"/\*([0-9a-f]{4,})\*/", l)
    if m3 and cur:
        amap[int(m3.group(1), 16)] = cur
rows = list(csv.reader(open(sass_csv)))
h = rows[1]
ia, iss, iex = h.index("Address"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
inn = h.index("Warp Stall Sampling (Not-issued Samples)")
base = int(rows[2][ia], 16)
agg = collections.defaultdict(lambda: [0.0, 0.0, 0.0])
tot = [0.0, 0.0, 0.0]
for r in rows[2:]:
    try:
        a = int(r[ia], 16) - base
        s, x, ni = float(r[iss] or 0), float(r[iex] or 0), float(r[inn] or 0)
    except ValueError:
        continue
    k = amap.get(a, ("?", 0))
    for j, val in enumerate((s, x, ni)):
        agg[k][j] += val
        tot[j] += val
src = {}
def text(f, n):
    import os
    p = os.path.join("paper_conf_ipps_mlakarwps21_b200/csrc", f)
    if p not in src:
        src[p] = open(p).read().splitlines() if os.path.exists(p) else []
    return src[p][n - 1].strip()[:70] if 0 < n <= len(src[p]) else ""
print(f"samples {tot[0]:.0f}  instructions {tot[1]:.0f}")
for title, j in (("by all stall samples", 0), ("by not-issued samples", 2), ("by instructions executed", 1)):
    print("top", title)
    for k, v in sorted(agg.items(), key=lambda t: -t[1][j])[:15]:
        print(f"  {100 * v[j] / max(tot[j], 1):5.1f}%  {k[0]}:{k[1]:<5d} {text(*k)}")

"""Aggregate an ncu source-page capture (cuda,sass) by match.cu function: instructions and stall samples.
    python scripts/src_regions.py gpurun_out/src_X.ncu-rep [top_lines]"""
import csv, re, subprocess, sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
src = open("paper_conf_icde_yuan0ha0024_b200/csrc/match.cu").read().splitlines()
starts = []
for i, l in enumerate(src, 1):
    m = re.match(r"^(?:template <[^>]*>\s*)?(?:__device__|__global__)[^(]*?(\w+)\(", l)
    if m:
        starts.append((i, m.group(1)))
def region(f, ln):
    if f != "match.cu":
        return f
    name = "top"
    for s, n in starts:
        if s <= ln:
            name = n
    return name
res, fn = [], None
for r in rows:
    if r and r[0] == "File Path":
        fn = r[1].split("/")[-1]
    if len(r) > 8 and r[0] not in ("", "Line No") and r[2] == "-":
        try:
            res.append((int(r[7]), int(r[4]), fn, int(r[0]), r[1].strip()[:100]))
        except ValueError:
            pass
tot = sum(x[0] for x in res) or 1
ts = sum(x[1] for x in res) or 1
agg = {}
for i, s, f, l, _ in res:
    k = region(f, l)
    a = agg.setdefault(k, [0, 0])
    a[0] += i
    a[1] += s
print(f"total warp instructions {tot:.4g}, stall samples {ts}")
for k, v in sorted(agg.items(), key=lambda x: -x[1][0]):
    print(f"  {k:28s} inst {100 * v[0] / tot:5.1f}%  stall {100 * v[1] / ts:5.1f}%")
print("top lines:")
for i, s, f, l, t in sorted(res, reverse=True)[:top]:
    print(f"  {100 * i / tot:5.2f}% inst {100 * s / ts:5.2f}% stall  {f}:{l}  {t}")

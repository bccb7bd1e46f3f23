"""Warp-stall samples of an ncu capture per CUDA source line (needs -lineinfo builds).
usage: python tools/ncu_lines.py <report.ncu-rep> <object.o> <kernel-substring> [top]
Maps each SASS address of the report's source page to the line nvdisasm -g attributes it to."""
import csv, io, os, re, subprocess, sys, tempfile, collections

rep, obj, kname = sys.argv[1], sys.argv[2], sys.argv[3]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h = rows[hdr]
ia, iw = h.index("Address"), h.index("Warp Stall Sampling (All Samples)")
samples = []
for r in rows[hdr + 1:]:
    if len(r) <= iw or not r[ia].startswith("0x"):
        continue
    samples.append((int(r[ia], 16), int(r[iw] or 0)))
base = samples[0][0]
tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=tmp, capture_output=True)
cubin = [f for f in os.listdir(tmp) if f.endswith(".cubin")][0]
sass = subprocess.run(["nvdisasm", "-g", os.path.join(tmp, cubin)], capture_output=True, text=True).stdout
lines = sass.splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith(".text.") and kname in l)
off2line, cur = {}, None
for l in lines[start + 1:]:
    if l.startswith(".text.") or l.startswith(".nv."):
        break
    m = re.search(r'//## File "([^"]+)", line (\d+)', l)
    if m:
        cur = (m.group(1), int(m.group(2)))
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", l)
    if m and cur:
        off2line[int(m.group(1), 16)] = cur
agg = collections.Counter()
for a, n in samples:
    agg[off2line.get(a - base, ("?", 0))] += n
tot = sum(agg.values())
src = {}
print(f"total samples {tot}")
for (f, ln), n in agg.most_common(top):
    if f not in src and os.path.exists(f):
        src[f] = open(f).read().splitlines()
    text = src.get(f, [""] * (ln + 1))[ln - 1].strip() if ln else ""
    print(f"{n:7d} {100.0 * n / tot:5.1f}%  {os.path.basename(f)}:{ln}  {text[:100]}")

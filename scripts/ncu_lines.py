"""Aggregate ncu warp-stall samples per CUDA source line.

usage: ncu_lines.py sass.csv kernel.cubin kernel_substring [top]
sass.csv = `ncu -i rep --page source --csv --print-source sass`; the cubin is
the one the report ran (cuobjdump -xelf all); line info needs -lineinfo.
"""
import csv, re, subprocess, sys, collections

sass_csv, cubin, kname = sys.argv[1:4]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 30
rows = list(csv.reader(open(sass_csv)))
hdr, data = rows[1], rows[2:]
i_s = hdr.index("Warp Stall Sampling (All Samples)")
stall = [j for j, h in enumerate(hdr) if h.startswith("stall") and "Not Issued" not in h]
base = int(data[0][0], 16)
dis = subprocess.run(["nvdisasm", "-g", "-c", cubin], capture_output=True, text=True).stdout
off2line, cur, inside, line = {}, None, False, None
for l in dis.splitlines():
    if l.startswith("//----") and ".text." in l:
        inside = kname in l
    if not inside:
        continue
    m = re.search(r'File "([^"]+)", line (\d+)', l)
    if "## File" in l and m:
        line = m.group(1).split("/")[-1] + ":" + m.group(2)
    m = re.match(r'\s*/\*([0-9a-f]{4,})\*/', l)
    if m and line is not None:
        off2line[int(m.group(1), 16)] = line
agg = collections.Counter()
why = collections.defaultdict(collections.Counter)
for r in data:
    if not r[i_s].isdigit():
        continue
    ln = off2line.get(int(r[0], 16) - base, "?")
    agg[ln] += int(r[i_s])
    for j in stall:
        if r[j].isdigit():
            why[ln][hdr[j]] += int(r[j])
tot = sum(agg.values())
print("total samples", tot)
for ln, v in agg.most_common(top):
    print(f"{v:7d} {100.0 * v / tot:5.1f}%  {ln:28s}  " + ", ".join(f"{k[6:]}={c}" for k, c in why[ln].most_common(2)))

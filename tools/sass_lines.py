"""Map an ncu source-page CSV (SASS addresses, warp-state samples) to CUDA source lines using
nvdisasm -g output of the same cubin: python tools/sass_lines.py all.sass kernel_substr src.csv [file_substr]"""
import csv, re, sys, collections
sass, kern, csvf = sys.argv[1], sys.argv[2], sys.argv[3]
fsub = sys.argv[4] if len(sys.argv) > 4 else ""
off2line, cur, inside, loc = {}, None, False, None
for L in open(sass):
    if L.startswith("//---------------------"):
        inside = kern in L
        continue
    if not inside:
        continue
    m = re.search(r'//## File "([^"]+)", line (\d+)', L)
    if m:
        loc = (m.group(1).split("/")[-1], int(m.group(2)))
        continue
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/", L)
    if m and loc:
        off2line[int(m.group(1), 16)] = loc
rows = list(csv.reader(open(csvf)))
hdr = rows[1]
ia, isamp = hdr.index("Address"), hdr.index("Warp Stall Sampling (All Samples)")
base = int(rows[2][ia], 16)
agg = collections.Counter()
tot = 0
for r in rows[2:]:
    try:
        a, s = int(r[ia], 16) - base, int(r[isamp])
    except (ValueError, IndexError):
        continue
    tot += s
    agg[off2line.get(a, ("?", 0))] += s
print("total samples", tot, "mapped offsets", len(off2line))
for (f, l), s in agg.most_common(60):
    if fsub in f:
        print("%8d %5.2f%%  %s:%d" % (s, 100.0 * s / tot, f, l))

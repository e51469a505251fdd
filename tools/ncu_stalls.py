"""Top SASS instructions by a stall reason from an ncu source page CSV.
usage: ncu -i rep --page source --csv --print-source sass > f.csv; python tools/ncu_stalls.py f.csv stall_dispatch [N]"""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
col = h.index(sys.argv[2]); src = h.index("Source"); addr = h.index("Address")
n = int(sys.argv[3]) if len(sys.argv) > 3 else 25
data = []
for r in rows[2:]:
    try:
        data.append((int(r[col] or 0), r[addr], r[src]))
    except (ValueError, IndexError):
        pass
tot = sum(d[0] for d in data)
print("total", tot)
by_op = collections.Counter()
for c, a, s in data:
    by_op[s.split()[0] if not s.startswith("@") else s.split()[1]] += c
print(by_op.most_common(12))
for c, a, s in sorted(data, reverse=True)[:n]:
    print(c, a, s[:90])

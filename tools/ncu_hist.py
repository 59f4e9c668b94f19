"""Execution-count classes of SASS instructions of an ncu report (which code regions run how often)."""
import csv, subprocess, io, collections, sys
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]; ix = {h: i for i, h in enumerate(hdr)}
data = [r for r in rows[2:] if len(r) == len(hdr) and r[0] != "Address"]
E = "Instructions Executed"
tot = sum(int(r[ix[E]] or 0) for r in data)
print("total executed", tot, "static instrs", len(data))
# contiguous regions with identical execution counts
regions = []
for r in data:
    e = int(r[ix[E]] or 0)
    if regions and regions[-1][0] == e:
        regions[-1][1] += 1; regions[-1][3] = r[ix["Address"]][-5:]
    else:
        regions.append([e, 1, r[ix["Address"]][-5:], r[ix["Address"]][-5:], r[ix["Source"]].strip()[:50]])
regions.sort(key=lambda x: -x[0] * x[1])
for e, n, a0, a1, src in regions[:int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    print(f"{a0}-{a1} count {e:8d} x {n:4d} = {e*n:10d} ({100*e*n/tot:5.1f}%)  {src}")

"""Per-region executed warp-instructions of an ncu report (source page, -lineinfo):
regions = line ranges of one file given as name=file:a-b ...; the rest is 'other'."""
import csv, io, subprocess, sys
rep = sys.argv[1]
regs = []
for a in sys.argv[2:]:
    name, rng = a.split("=")
    f, ab = rng.split(":")
    lo, hi = ab.split("-")
    regs.append((name, f, int(lo), int(hi)))
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows, f, hdr = [], None, None
for r in csv.reader(io.StringIO(out)):
    if len(r) == 2 and r[0] == "File Path": f = r[1].split("/")[-1]; continue
    if len(r) == 2: continue
    if r and r[0] == "Line No": hdr = r; continue
    if hdr and r and r[0]:
        try: rows.append((f, int(r[0]), int(r[7]), int(r[8]) if len(r) > 8 and r[8].isdigit() else 0))
        except ValueError: pass
tot = sum(r[2] for r in rows)
acc = {}
for f, ln, ex, th in rows:
    key = "other:" + f
    for name, rf, lo, hi in regs:
        if f == rf and lo <= ln <= hi:
            key = name
            break
    a = acc.setdefault(key, [0, 0])
    a[0] += ex
    a[1] += th
print("total warp-instructions", tot)
for k, (ex, th) in sorted(acc.items(), key=lambda x: -x[1][0]):
    print(f"{k:28s} {ex:>10} {100*ex/tot:5.1f}%  thr/instr {th/ex if ex and th else 0:5.1f}")

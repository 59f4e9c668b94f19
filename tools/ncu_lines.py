"""Per-source-line executed instructions of an ncu report (cuda,sass view; needs -lineinfo)."""
import csv, io, subprocess, sys
rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows, f, hdr = [], None, None
for r in csv.reader(io.StringIO(out)):
    if len(r) == 2 and r[0] == "File Path": f = r[1].split("/")[-1]; continue
    if len(r) == 2: continue
    if r and r[0] == "Line No": hdr = r; continue
    if hdr and r and r[0]:
        try: rows.append((int(r[7]), int(r[4]), f, int(r[0]), r[1].strip()[:90]))
        except ValueError: pass
tot = sum(r[0] for r in rows)
print("total", tot)
for r in sorted(rows, reverse=True)[:n]:
    print(f"{r[0]:>9} {100*r[0]/tot:5.1f}%  smp {r[1]:>4}  {r[2]}:{r[3]}  {r[4]}")

"""Per-region warp instructions and SIMT efficiency (thread instr / warp instr) of an ncu
report, regions = line ranges of event_kernel.cuh given as name:lo-hi arguments."""
import csv, io, subprocess, sys
rep = sys.argv[1]
regions = [(a.split(":")[0], *map(int, a.split(":")[1].split("-"))) for a in sys.argv[2:]]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
f, hdr, rows = None, None, []
for r in csv.reader(io.StringIO(out)):
    if len(r) == 2 and r[0] == "File Path": f = r[1].split("/")[-1]; continue
    if len(r) == 2: continue
    if r and r[0] == "Line No": hdr = r; continue
    if hdr and r and r[0]:
        try: rows.append((f, int(r[0]), int(r[7]), int(r[8])))
        except ValueError: pass
tot_w = sum(x[2] for x in rows); tot_t = sum(x[3] for x in rows)
print(f"total warp-instr {tot_w}  threads/instr {tot_t / max(tot_w, 1):.1f}")
for name, lo, hi in regions:
    w = sum(x[2] for x in rows if x[0] == "event_kernel.cuh" and lo <= x[1] <= hi)
    t = sum(x[3] for x in rows if x[0] == "event_kernel.cuh" and lo <= x[1] <= hi)
    print(f"{name:16s} warp-instr {w:9d} ({100 * w / tot_w:5.1f}%)  threads/instr {t / max(w, 1):5.1f}")
other = [x for x in rows if x[0] != "event_kernel.cuh"]
w = sum(x[2] for x in other); t = sum(x[3] for x in other)
print(f"{'other files':16s} warp-instr {w:9d} ({100 * w / tot_w:5.1f}%)  threads/instr {t / max(w, 1):5.1f}")

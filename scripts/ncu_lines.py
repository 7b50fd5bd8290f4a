"""Per-CUDA-source-line stall samples from an ncu report (builder tooling)."""
import csv, io, subprocess, sys
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
res = []
cur_file = None
for r in rows:
    if r and r[0] == "File Path":
        cur_file = r[1].split("/")[-1]
        continue
    if len(r) > 6 and r[0].isdigit() and r[2] == "-":
        res.append((int(r[4] or 0), cur_file, int(r[0]), r[1].strip()))
tot = sum(x[0] for x in res) or 1
for s, f, ln, src in sorted(res, reverse=True)[: int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    print(f"{100 * s / tot:5.1f}%  {f}:{ln:<5d} {src[:100]}")

"""Per-CUDA-source-line stall samples / executed instructions of one kernel in an
ncu report (diagnostic):  python scripts/ncu_lines.py report.ncu-rep [top]"""
import csv, io, subprocess, sys
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
lines = []
for r in rows[3:]:
    if r and r[0].strip():
        try:
            lines.append((int(r[0]), r[1].strip()[:100], float(r[4]), float(r[7])))
        except ValueError:
            pass
ts = sum(l[2] for l in lines) or 1
ti = sum(l[3] for l in lines) or 1
print(f"samples {ts:.0f}  warp-instructions {ti:.3g}")
for ln, s, smp, ins in sorted(lines, key=lambda x: -x[2])[:top]:
    print(f"{ln:5d} {100 * smp / ts:5.1f}% samp {100 * ins / ti:5.1f}% inst | {s}")

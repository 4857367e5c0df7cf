"""Per-source-line totals from `ncu -i R --page source --csv --print-source cuda,sass` (stdin):
instructions executed, thread instructions, stall samples.  Usage: ... | python scripts/ncu_lines.py [top]"""
import csv
import sys

top = int(sys.argv[1]) if len(sys.argv) > 1 else 40
rows = list(csv.reader(sys.stdin))
fn, cur, hdr, lines = None, None, None, {}
for r in rows:
    if not r:
        continue
    if r[0] in ("File Path", "Function Name"):
        if r[0] == "File Path":
            fn = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None:
        continue
    if r[0]:
        cur = (fn, int(r[0]), r[1].strip()[:70])
        d = dict(zip(hdr[2:], r[2:]))

        def f(k):
            try:
                return float(d.get(k, "0").replace(",", ""))
            except ValueError:
                return 0.0
        lines[cur] = [f("Instructions Executed"), f("Thread Instructions Executed"),
                      f("Warp Stall Sampling (All Samples)")]
tot = [sum(v[k] for v in lines.values()) for k in range(3)]
print(f"total warp inst {tot[0]:.3e}  thread inst {tot[1]:.3e}  samples {tot[2]:.0f}")
print(f"{'file:line':28s} {'inst%':>6s} {'thr/inst':>8s} {'samp%':>6s}  source")
for k, v in sorted(lines.items(), key=lambda kv: -kv[1][2])[:top]:
    print(f"{k[0][:20] + ':' + str(k[1]):28s} {100 * v[0] / tot[0]:6.2f} {v[1] / max(v[0], 1):8.1f} "
          f"{100 * v[2] / tot[2]:6.2f}  {k[2]}")

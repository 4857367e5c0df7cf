"""Warp instructions and stall samples of an ncu source page, grouped by the function of
fill2_impl.cuh each source line belongs to (found from the source text ncu embeds, so the
grouping always matches the profiled build).  Usage: python scripts/ncu_funcs.py REPORT"""
import csv
import io
import re
import subprocess
import sys

DEF = re.compile(r"^(?:template\s*<[^>]*>\s*)?(?:__device__|__global__|__host__)[\w\s:<>,*&()]*?"
                 r"\b(\w+)\s*\(")
# named sub-regions inside the kernel body (comments that start a phase)
PHASES = [("---- seed", "kernel: seed"), ("---- thresholds in increasing order", "kernel: windows"),
          ("---- U part, diagonal", "kernel: U part / stage / emit"),
          ("for (;;) {", None)]


def main():
    out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv",
                          "--print-source", "cuda,sass"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, fname, acc = None, "", {}
    tot_i = tot_s = 0.0
    func = "?"
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].split("/")[-1]
            func = "?"
        elif r[0] == "Line No":
            hdr = r
        elif hdr and r[0].isdigit():
            d = dict(zip(hdr[2:], r[2:]))
            src = r[1]
            if fname == "fill2_impl.cuh":
                m = DEF.match(src.strip())
                if m and not src.startswith(" "):
                    func = m.group(1)
                for key, name in PHASES:
                    if name and key in src and func == "fill2_kernel":
                        func = "fill2_kernel"
                        sub = name
                        acc.setdefault("_sub", {})
                        d["_sub"] = sub
                        globals()["_cur_sub"] = sub
            try:
                i = float(d.get("Instructions Executed") or 0)
                s = float(d.get("Warp Stall Sampling (All Samples)") or 0)
            except ValueError:
                continue
            tot_i += i
            tot_s += s
            if fname == "fill2_impl.cuh":
                name = func
                if func == "fill2_kernel":
                    name = globals().get("_cur_sub", "kernel: setup/claim")
            else:
                name = fname
            a = acc.setdefault(name, [0.0, 0.0])
            a[0] += i
            a[1] += s
    acc.pop("_sub", None)
    print(f"total warp instructions {tot_i:.4e}, stall samples {tot_s:.0f}")
    for k, (i, s) in sorted(acc.items(), key=lambda x: -x[1][0]):
        print(f"  {k:40s} inst {i / tot_i * 100:6.2f}%  samples {s / tot_s * 100:6.2f}%")


if __name__ == "__main__":
    main()

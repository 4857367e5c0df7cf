"""Group the per-line output of scripts/ncu_hot.py (captured on this source tree) by the
fill2_impl.cuh function each line belongs to, and by phase inside fill2_kernel.
Usage: python scripts/hot_funcs.py HOT_TXT [warp_inst_per_sv]"""
import re
import sys

SRC = "paper_conf_ppopp_xia0ar23_b200/csrc/fill2_impl.cuh"


def main():
    src = open(SRC).read().split("\n")
    starts, phases = [], []
    for k, line in enumerate(src, start=1):
        m = re.match(r"^(?:__device__|__global__|__host__ __device__)[^(]*?\b(\w+)\s*\(", line)
        if m:
            starts.append((k, m.group(1)))
        if re.match(r"^\s+fill2_kernel\(", line):
            starts.append((k, "fill2_kernel"))
        for key, name in (("---- seed", "kernel: seed"),
                          ("---- thresholds in increasing order", "kernel: threshold windows"),
                          ("---- U part, diagonal", "kernel: U part / stage / emit")):
            if key in line:
                phases.append((k, name))

    def func(ln):
        f = "file scope"
        for k, n in starts:
            if k <= ln:
                f = n
        if f == "fill2_kernel":
            f = "kernel: setup / row claim"
            for k, n in phases:
                if k <= ln:
                    f = n
        return f

    acc, tot = {}, 0.0
    for line in open(sys.argv[1]).read().split("\n"):
        m = re.match(r"\s*([\d.]+)% samp\s+([\d.]+)% inst\s+(\S+):(\d+)", line)
        if not m:
            continue
        samp, inst, f, ln = float(m.group(1)), float(m.group(2)), m.group(3), int(m.group(4))
        name = func(ln) if f == "fill2_impl.cuh" else f
        a = acc.setdefault(name, [0.0, 0.0])
        a[0] += inst
        a[1] += samp
        tot += inst
    per_sv = float(sys.argv[2]) if len(sys.argv) > 2 else None
    print(f"lines listed cover {tot:.1f}% of the warp instructions")
    for k, (i, s_) in sorted(acc.items(), key=lambda x: -x[1][0]):
        extra = f"  {i / 100 * per_sv:5.2f} warp inst / SV" if per_sv else ""
        print(f"  {k:32s} inst {i:6.2f}%  samples {s_:6.2f}%{extra}")


if __name__ == "__main__":
    main()

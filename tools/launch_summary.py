"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) into
per-kernel shares; FT2 kernels (libft2.so) are marked.
python tools/launch_summary.py launches.csv"""
import collections
import csv
import sys


def main(path):
    rows = [r for r in csv.reader(l for l in open(path) if l.startswith('"'))]
    hdr = rows[0]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    tot = collections.Counter()
    cnt = collections.Counter()
    for r in rows[1:]:
        if r[mi] != "gpu__time_duration.sum":
            continue
        name = r[ki]
        if "ft2impl::" in name or name.startswith("void ft2impl") or "gemm_kernel<" in name and "ft2" in name:
            name = "FT2 " + name.split("ft2impl::", 1)[1].split("(")[0]
        tot[name] += float(r[vi].replace(",", "")) / 1e3
        cnt[name] += 1
    all_us = sum(tot.values())
    print(f"launches: {sum(cnt.values())}   summed kernel time: {all_us / 1e3:.2f} ms")
    print("  share    total_us  count   avg_us  kernel")
    for n, t in tot.most_common():
        print(f"{100 * t / all_us:6.2f}%  {t:10.1f}  {cnt[n]:5d}  {t / cnt[n]:7.2f}  {n[:90]}")
    ft = sum(t for n, t in tot.items() if n.startswith("FT2 "))
    print(f"FT2 kernels (libft2.so) total share: {100 * ft / all_us:.2f}%  ({ft / 1e3:.2f} ms)")


if __name__ == "__main__":
    main(sys.argv[1])

"""Summarise an ncu launch list (gpu__time_duration.sum) into per-kernel shares of
the last outer iteration of a bench run (cold-cache, serialised: compare shares)."""
import collections
import csv
import sys


def main(path, out=None, nmodes_arg=None):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    hdr, data = rows[0], rows[1:]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    launches = [(r[ki], float(r[vi].replace(",", ""))) for r in data if r[mi] == "gpu__time_duration.sum"]
    starts = [i for i, (k, _) in enumerate(launches) if "k_chol_inverse" in k]
    # the last outer iteration starts at the N-th last chol_inverse (one per mode)
    nmodes = min(int(nmodes_arg), len(starts)) if nmodes_arg else min(3, len(starts))
    text = []
    tot = collections.Counter()
    first = starts[-nmodes] if nmodes else 0
    for k, t in launches[first:]:
        name = k.split("(")[0].replace("void ", "").replace("cstf::<unnamed>::", "").split("<")[0]
        tot[name] += t
    s = sum(tot.values())
    text.append(f"{path}: {len(launches)} launches; from the {nmodes}-th last k_chol_inverse to the end")
    for k, t in tot.most_common():
        text.append(f"  {k:28s} {t / 1e3:10.3f} us  {100 * t / s:5.1f}%")
    text.append(f"  total {s / 1e3:.3f} us")
    print("\n".join(text))
    if out:
        open(out, "w").write("\n".join(text) + "\n")


if __name__ == "__main__":
    # usage: launch_summary.py launches.csv [out.txt] [nmodes]
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None, sys.argv[3] if len(sys.argv) > 3 else None)

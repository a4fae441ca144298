"""Per-launch table of an ncu --metrics CSV (time, DRAM bytes, L2 hit rate,
SM throughput), restricted to the last training step (launches after the
last 'k_xent' minus the forward): prints every launch of the last epoch."""
import collections
import csv
import sys


def load(path):
    rows = list(csv.DictReader(l for l in open(path) if not l.startswith("==")))
    by = collections.OrderedDict()
    for r in rows:
        by.setdefault(int(r["ID"]), {"name": r["Kernel Name"]})[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
    return by


def main(path, first_kernel="k_gemm_nt_p", steps=2):
    by = load(path)
    ids = sorted(by)
    # the last `1/steps` of the wg launches are the last epoch
    wg = [i for i in ids if "wg::" in by[i]["name"] or "unnamed>::" in by[i]["name"]]
    last = wg[len(wg) // steps * (steps - 1):] if steps > 1 else wg
    tot_t = tot_b = 0.0
    for i in last:
        m = by[i]
        t = m["gpu__time_duration.sum"] / 1e3
        b = (m["dram__bytes_read.sum"] + m["dram__bytes_write.sum"]) / 1e9
        tot_t += t
        tot_b += b
        nm = m["name"].replace("wg::(anonymous namespace)::", "").replace("unnamed>::", "").replace("void ", "")[:58]
        print("%4d %-58s %8.1f us %6.2f GB %5.2f TB/s L2hit %5.1f sm %5.1f" % (
            i, nm, t, b, b / t * 1e3 if t else 0, m.get("lts__t_sector_hit_rate.pct", 0),
            m.get("sm__throughput.avg.pct_of_peak_sustained_elapsed", 0)))
    print("total %.3f ms  %.2f GB" % (tot_t / 1e3, tot_b))


if __name__ == "__main__":
    main(sys.argv[1], steps=int(sys.argv[2]) if len(sys.argv) > 2 else 2)

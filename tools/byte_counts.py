"""Per-call DRAM bytes of every variant from ncu launch lists (Table I /
Lemmas 2-5, Theorems 6-7 byte counts, SURVEY 4 'byte counts per element
checked against ncu DRAM bytes').

python tools/byte_counts.py gpurun_out/bytes_<variant>.csv ...   (here, on the CSVs)
On the box: ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum
  --clock-control none -k regex:sat_ --csv --log-file X.csv python tools/prof_one.py cfg3b 0 2 <variant>
"""
import csv
import sys

ALG = {"1r1w": 2, "2r2w": 4, "2r1w": 3, "1+rr1w": None, "4r4w": 8}   # x eb x n x m


def main():
    n = 16384 * 16384
    eb = 4
    for path in sys.argv[1:]:
        rows = list(csv.reader(open(path)))
        h = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
        hdr = rows[h]
        tot = {"dram__bytes_read.sum": 0.0, "dram__bytes_write.sum": 0.0, "gpu__time_duration.sum": 0.0}
        kernels = set()
        unit = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
                "msecond": 1e-3, "ns": 1e-9, "us": 1e-6, "ms": 1e-3}
        ids = set()
        for r in rows[h + 1:]:
            d = dict(zip(hdr, r))
            if d.get("Metric Name") in tot:
                tot[d["Metric Name"]] += float(d["Metric Value"].replace(",", "")) * unit.get(d["Metric Unit"], 1)
                kernels.add(d["Kernel Name"].split("<")[0].replace("void ", ""))
                ids.add(d["ID"])
        variant = path.rsplit("_", 1)[-1].replace(".csv", "")
        calls = 2
        rd, wr = tot["dram__bytes_read.sum"] / calls, tot["dram__bytes_write.sum"] / calls
        alg = ALG.get(variant)
        print(f"{variant:7s} launches/call {len(ids) // calls:3d}  DRAM read {rd / 1e9:.3f} GB + write {wr / 1e9:.3f} GB"
              f" = {(rd + wr) / (eb * n):.2f} x eb x n^2" + (f"  (Table I: {alg})" if alg else "  (Table I: 2 + r)")
              + f"  kernels {sorted(kernels)}")


if __name__ == "__main__":
    main()

"""Summarise an ncu report (--set full) of k_spmm into profiles/: key metrics per
launch, and the DRAM traffic per step that bench.py reports as roofline.traffic.

  python tools/ncu_summary.py gpurun_out/X.ncu-rep TAG [--workload c2] [--launches-per-step 1]
"""
import argparse
import csv
import io
import json
import os
import subprocess

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "l1tex__m_xbar2l1tex_read_bytes.sum",
        "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed"]
TO_BYTES = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("tag")
    ap.add_argument("--workload", default="c2")
    ap.add_argument("--launches-per-step", type=int, default=1)
    a = ap.parse_args()
    raw = subprocess.run(["ncu", "-i", a.rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    out = []
    for d in data:
        rec = {"kernel": d[hdr.index("Kernel Name")][:80]}
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                v = d[i].replace(",", "")
                try:
                    x = float(v)
                except ValueError:
                    x = v
                if isinstance(x, float) and units[i] in TO_BYTES:
                    x *= TO_BYTES[units[i]]
                    rec[k + " [B]"] = x
                else:
                    rec[k + (f" [{units[i]}]" if units[i] else "")] = x
        out.append(rec)
    os.makedirs("profiles", exist_ok=True)
    with open(f"profiles/{a.tag}_ncu_summary.json", "w") as f:
        json.dump(out, f, indent=1)
    spmm = [r for r in out if "k_spmm" in r["kernel"]]
    if spmm:
        traffic = sum(r.get("dram__bytes_read.sum [B]", 0) + r.get("dram__bytes_write.sum [B]", 0)
                      for r in spmm) / len(spmm)
        path = "profiles/ncu_traffic.json"
        try:
            allw = json.load(open(path))
            if "workload" in allw:      # old single-entry format
                allw = {allw["workload"]: allw}
        except Exception:
            allw = {}
        allw[a.workload] = {"bytes_per_step": traffic * a.launches_per_step, "bytes_per_launch": traffic,
                            "source": f"{os.path.basename(a.rep)} (ncu --set full, {len(spmm)} k_spmm "
                                      "launches, dram__bytes_read.sum + dram__bytes_write.sum)"}
        json.dump(allw, open(path, "w"), indent=1)
    for r in out:
        print(json.dumps(r))


if __name__ == "__main__":
    main()

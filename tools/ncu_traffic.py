"""ncu DRAM traffic of the dominant kernels of bench.py, hash-stamped.

    python tools/ncu_traffic.py            # on a GPU box: captures c2 and c3, writes
                                           # profiles/ncu_traffic.json (+ the raw CSVs)
    python tools/ncu_traffic.py case c2    # the workload one capture profiles

Each case runs the exact call bench.py times (same shape, dtype, kind, AUTO dispatch,
out-of-place), warms up, and ncu (`--set full --clock-control none`) captures one launch of
the dominant kernel (cold caches: ncu flushes between replays).  The JSON records
dram__bytes_read.sum / dram__bytes_write.sum / gpu__time_duration.sum per launch and the
sha256 of the library sources (bench.source_sha256); bench.py reports the traffic only while
that hash matches the sources it runs.
"""
import csv
import datetime
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

CASES = {
    # name: (kernel regex, dtype, G, N, dist, kind)
    "c2": ("chunk_scan_kernel", "i32", 4096, 1 << 14, "i32", "inclusive"),
    "c3": ("lookback_l2_kernel", "f32", 1, 1 << 30, "f32u", "inclusive"),
}
METRICS = ["dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum"]


def run_case(name):
    import torch
    import inputs
    import paper_conf_ipps_dieguezadnm18_b200 as sb
    _, dt, G, N, dist, kind = CASES[name]
    t = torch.empty(G * N, dtype=torch.int32, device="cuda")
    inputs.fill_device(t, dist, 0x5CA2018 + (2 if name == "c2" else 3))
    x = t.view({"i32": torch.int32, "f32": torch.float32}[dt]).view(G, N)
    y = torch.empty_like(x)
    for _ in range(4):
        sb.scan(x, "add", kind, out=y)
    torch.cuda.synchronize()


def capture(name, outdir):
    kern = CASES[name][0]
    csv_path = os.path.join(outdir, "ncu_traffic_%s.csv" % name)
    cmd = ["ncu", "--set", "full", "--clock-control", "none", "--kernel-name", "regex:" + kern,
           "--launch-skip", "2", "--launch-count", "1", "--csv", "--page", "raw",
           "--metrics", ",".join(METRICS), sys.executable, os.path.abspath(__file__), "case", name]
    r = subprocess.run(cmd, capture_output=True, text=True)
    open(csv_path, "w").write(r.stdout)
    if r.returncode != 0:
        raise RuntimeError("ncu failed for %s:\n%s" % (name, r.stderr[-3000:]))
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith('"')]
    rows = list(csv.reader(io.StringIO("\n".join(lines))))
    hdr = rows[0]
    data = [row for row in rows[2:] if len(row) == len(hdr)] or [row for row in rows[1:] if len(row) == len(hdr)]
    rec = dict(zip(hdr, data[-1]))

    def num(key):
        v = rec[key].replace(",", "")
        return float(v)
    units = dict(zip(hdr, rows[1])) if len(rows) > 1 else {}
    scale = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}
    out = {"kernel": rec.get("Kernel Name", kern)}
    for m in METRICS[:2]:
        out[m.split(".")[0].replace("dram__", "dram_") ] = num(m) * scale.get(units.get(m, "byte"), 1.0)
    tu = units.get(METRICS[2], "nsecond")
    out["duration_us"] = num(METRICS[2]) * {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3}.get(tu, 1e-3)
    return out


def main():
    if len(sys.argv) > 2 and sys.argv[1] == "case":
        run_case(sys.argv[2])
        return
    import bench
    outdir = os.path.join(ROOT, "gpurun_out")
    os.makedirs(outdir, exist_ok=True)
    res = {"src_sha256": bench.source_sha256(),
           "captured": datetime.datetime.now(datetime.timezone.utc).strftime("%Y-%m-%dT%H:%MZ"),
           "how": "ncu --set full --clock-control none, one launch after 2 warm-up launches, cold caches",
           "cases": {}}
    for name in CASES:
        c = capture(name, outdir)
        _, dt, G, N, _, _ = CASES[name]
        c["algorithmic_bytes"] = 8.0 * G * N
        c["dram_bytes_read"] = c.pop("dram_bytes_read")
        c["dram_bytes_write"] = c.pop("dram_bytes_write")
        c["traffic_over_algorithmic"] = (c["dram_bytes_read"] + c["dram_bytes_write"]) / c["algorithmic_bytes"]
        res["cases"][name] = c
        print(name, json.dumps(c), flush=True)
    json.dump(res, open(os.path.join(ROOT, "profiles", "ncu_traffic.json"), "w"), indent=1)
    json.dump(res, open(os.path.join(outdir, "ncu_traffic.json"), "w"), indent=1)


if __name__ == "__main__":
    main()

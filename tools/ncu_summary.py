"""Summarises ncu output brought back in gpurun_out/ into tracked JSON under profiles/.

  python tools/ncu_summary.py --round 1
reads gpurun_out/launches.csv (the --metrics gpu__time_duration.sum launch list), gpurun_out/mover.ncu-rep
and gpurun_out/scan.ncu-rep (--set full captures) and writes profiles/r01_launches.json,
profiles/r01_mover_ncu.json, profiles/r01_scan_ncu.json and profiles/mover_ncu.json (read by bench.py for
roofline.traffic)."""
import argparse
import csv
import io
import json
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
NCU = "/usr/local/cuda/bin/ncu"

RAW = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
       "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
       "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
       "launch__grid_size", "launch__block_size", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
       "lts__t_sector_hit_rate.pct", "l1tex__m_l1tex2xbar_req_cycles_active_op_tma.sum",
       "smsp__inst_executed.sum", "launch__shared_mem_per_block_dynamic", "pcie__read_bytes.sum",
       "pcie__write_bytes.sum"]


def raw_metrics(rep):
    out = subprocess.run([NCU, "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return {}
    h, units, v = rows[0], rows[1], rows[2]
    d = {"kernel": v[h.index("Kernel Name")] if "Kernel Name" in h else None}
    for k in RAW:
        if k in h:
            i = h.index(k)
            d[k] = {"value": v[i], "unit": units[i]}
    stalls = {}
    for i, k in enumerate(h):
        if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued"):
            try:
                x = float(v[i].replace(",", ""))
            except ValueError:
                continue
            if x > 0:
                stalls[k.replace("smsp__pcsamp_warps_issue_stalled_", "")] = x
    tot = sum(stalls.values()) or 1
    d["stall_samples_share"] = {k: round(x / tot, 3) for k, x in sorted(stalls.items(), key=lambda t: -t[1])[:8]}
    return d


def to_bytes(m):
    v = float(m["value"].replace(",", ""))
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(m["unit"], 1)


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr, tot = None, {}
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            name = d["Kernel Name"].split("(")[0].replace("(anonymous namespace)::", "")
            v = float(d["Metric Value"].replace(",", ""))
            t = tot.setdefault(name, [0.0, 0])
            t[0] += v
            t[1] += 1
    s = sum(v[0] for v in tot.values()) or 1
    return {k: {"launches": v[1], "total_ns": v[0], "share": round(v[0] / s, 4)}
            for k, v in sorted(tot.items(), key=lambda t: -t[1][0])}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--round", type=int, default=1)
    a = ap.parse_args()
    tag = f"r{a.round:02d}"
    os.makedirs(PROF, exist_ok=True)
    for lst in ("launches", "bench_launches", "smoke_launches"):
        if os.path.exists(os.path.join(OUT, f"{lst}.csv")):
            json.dump(launches(os.path.join(OUT, f"{lst}.csv")), open(os.path.join(PROF, f"{tag}_{lst}.json"), "w"),
                      indent=1)
    for name in ("mover", "scan", "walk", "emit", "front"):
        rep = os.path.join(OUT, f"{name}.ncu-rep")
        if not os.path.exists(rep):
            continue
        d = raw_metrics(rep)
        if name == "mover" and "dram__bytes_read.sum" in d:
            d["dram_bytes_per_launch"] = to_bytes(d["dram__bytes_read.sum"]) + to_bytes(d["dram__bytes_write.sum"])
            json.dump({"dram_bytes_per_launch": d["dram_bytes_per_launch"], "source": f"profiles/{tag}_mover_ncu.json"},
                      open(os.path.join(PROF, "mover_ncu.json"), "w"), indent=1)
        json.dump(d, open(os.path.join(PROF, f"{tag}_{name}_ncu.json"), "w"), indent=1)
        print(name, json.dumps(d)[:600])
    host = os.path.join(OUT, "host_step_metrics.csv")
    if os.path.exists(host):
        d = host_step(host)
        json.dump(d, open(os.path.join(PROF, f"{tag}_host_step_ncu.json"), "w"), indent=1)
        print("host step", json.dumps(d)[:600])


def host_step(path):
    """tools/gpu_ncu_host.sh: per kernel of one zero-copy server step (rings in pinned host memory), the
    PCIe bytes against the wire bytes the step must move (profile_step.py --host prints them)."""
    out = {}
    for r in csv.reader(open(path)):
        if len(r) < 15 or r[0] == "ID":
            continue
        k = r[4].split("(")[0].replace("unnamed>::", "")
        out.setdefault(k, {})[r[12]] = r[14]
    log = os.path.join(OUT, "ncu_host.log")
    if os.path.exists(log):
        for line in open(log):
            if line.startswith("{") and "wire_in" in line:
                out["step"] = json.loads(line)
    out["note"] = ("pcie__read_bytes / pcie__write_bytes are link-level counts (they include TLP protocol "
                   "overhead); compare them with the step's wire_in / reply_wire")
    return out


if __name__ == "__main__":
    main()

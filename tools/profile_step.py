"""Runs the bench workload's server step under the CUDA profiler window only (for ncu with
--profile-from-start off): endpoint setup (ring filling) is outside the window.

  ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
      --log-file gpurun_out/launches.csv python tools/profile_step.py --steps 3
  ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:mover \
      -c 1 -o gpurun_out/mover python tools/profile_step.py --steps 1
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_sc_eilingkkflm23_b200 import build, crk, workload  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--host", action="store_true")
    ap.add_argument("--streams", type=int, default=16)
    ap.add_argument("--payload-mib", type=int, default=64)
    ap.add_argument("--ctx", default="", help="crk_config overrides, e.g. mover_run=32,mover_reserve_ctas=16")
    a = ap.parse_args()
    build.build()
    dev = torch.device("cuda:0")
    ctx = crk.Context(0, **{k: int(v, 0) for k, v in (kv.split("=") for kv in a.ctx.split(",") if kv)})
    ep = workload.c5_endpoint(ctx, 0, dev, n_streams=a.streams, payload_per_stream=a.payload_mib << 20,
                              host_rings=a.host)
    idx = ctx.index(max_rings=a.streams, max_frags=1 << 20, max_records=1 << 14)
    workload.serve_step(idx, ep)  # warm
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    for _ in range(a.steps):
        workload.serve_step(idx, ep)
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    print(workload.check_results(idx, ep))
    print(json.dumps({"wire_in": ep.wire_in, "reply_wire": ep.reply_wire, "h2d_payload": ep.h2d_payload,
                      "d2h_payload": ep.d2h_payload, "host_rings": a.host, "steps_profiled": a.steps}))


if __name__ == "__main__":
    main()

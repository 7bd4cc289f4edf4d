"""e2e rate of the bench step (configs[1] through scan_batch_host, pinned buffers) for the
current SCANB200_HOST_PIECE / SCANB200_HOST_SLOTS settings: one JSON line."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_ipps_dieguezadnm18_b200 as sb  # noqa: E402

r = bench.e2e(sb, 1, K=5)
print(json.dumps({"piece": os.environ.get("SCANB200_HOST_PIECE"), "slots": os.environ.get("SCANB200_HOST_SLOTS"),
                  "Gelem/s": r["value"], "frac": r["frac_of_pcie_ceiling"],
                  "ceiling_GBs": r["pcie_ceiling"]["GB/s_each_way"]}), flush=True)

"""Short rows (N < 1024, and a few just above): packed_warp (span targets) vs the
one-tile-per-CTA look-back (variant 2) and the warp cascade, ~1 GiB of int32 per shape
(G = 2^28/N as in the paper's sweep), device time per call."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import inputs
import paper_conf_ipps_dieguezadnm18_b200 as sb
x = torch.empty(1 << 28, dtype=torch.int32, device="cuda")
inputs.fill_device(x, "i32", 3)
y = torch.empty_like(x)
def t(xv, yv, algo, param):
    for _ in range(2):
        sb.scan(xv, "add", out=yv, algo=algo, param=param)
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); s0.record()
    for _ in range(8):
        sb.scan(xv, "add", out=yv, algo=algo, param=param)
    s1.record(); torch.cuda.synchronize()
    return s0.elapsed_time(s1) / 8
PEAK = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6455.6
def main():
  for N in [1, 2, 3, 4, 8, 16, 32, 64, 100, 128, 255, 256, 257, 512, 600, 1000, 1023, 1024, 2048]:
      G = (1 << 28) // N
      xv, yv = x[:G * N].view(G, N), y[:G * N].view(G, N)
      res = []
      for algo, param in [("packed_warp", -1), ("packed_warp", 1024), ("packed_warp", 4096),
                          ("lookback", 2), ("lookback", 3), ("cascade_warp", -1)]:
          if algo == "cascade_warp" and N < 64:
              continue
          ms = t(xv, yv, algo, param)
          res.append("%s/%d %.1f%%" % (algo, param, 100 * 8 * G * N / ms / 1e6 / PEAK))
      print("N=%d G=%d auto=%s  " % (N, G, sb.plan(xv)[0]) + "  ".join(res), flush=True)


if __name__ == "__main__":
    main()

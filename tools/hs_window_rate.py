"""HotSpot leaf rate on one ~8704^2 window (the out-of-core plan's window size),
8 iterations per launch, under the conditions of the out-of-core run:
  aligned   window at a 128-B aligned base (ld = 8704)
  shifted   the same window 8 rows / 8 columns into a larger buffer (the plan's
            ping-pong windows shift by the iteration count each launch)
  copies    aligned, while pinned H2D and D2H copies run on two other streams
Cell updates per second of the valid region."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chey19_b200 as nu

S = int(os.environ.get("HS_S", "8704"))
LD = S + 64
R = C = 65536
big_t = torch.rand(S + 64, LD, device="cuda") * 10 + 330
big_p = torch.rand(S + 64, LD, device="cuda") * 0.5
big_o = torch.empty_like(big_t)


def views(sh):
    return [x[sh:sh + S, sh:sh + S] for x in (big_t, big_p, big_o)]


def rate(t, p, o, n=40, side=None):
    for _ in range(3):
        nu.hotspot_leaf(t, p, o, 8, gy0=1024, gx0=1024, rows=R, cols=C)
    torch.cuda.synchronize()
    if side:
        side()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(n):
        nu.hotspot_leaf(t, p, o, 8, gy0=1024, gx0=1024, rows=R, cols=C)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / n
    return {"ms": round(ms, 4), "gcups_valid": round((S - 16) ** 2 * 8 / ms / 1e6, 1)}


res = {"S": S}
res["aligned"] = rate(*views(0))
for sh in (4, 8, 32):
    res[f"shifted{sh}"] = rate(*views(sh))
hin = torch.empty(1 << 30, dtype=torch.uint8, pin_memory=True)
hout = torch.empty(1 << 30, dtype=torch.uint8, pin_memory=True)
din = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
dout = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def side():
    for _ in range(2):
        with torch.cuda.stream(s1):
            din.copy_(hin, non_blocking=True)
        with torch.cuda.stream(s2):
            hout.copy_(dout, non_blocking=True)


res["copies"] = rate(*views(0), side=side)
torch.cuda.synchronize()
print(json.dumps(res), flush=True)

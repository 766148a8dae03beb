"""One out-of-core HotSpot block's leaf sequence in isolation: 32 launches of 8
iterations on an interior 8704^2 window shrinking by 8 per side per launch,
ping-ponging between two window buffers in one arena (the plan's layout),
(a) alone, (b) while H2D / D2H copies of other slots run, as in the plan.
Compared with 32 launches on a fixed 8704^2 window."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chey19_b200 as nu

W, H, LI = 8704, 256, 8
R = C = 32768
gy, gx = 8192 - H, 8192 - H                      # an interior block's window origin
arena = torch.empty(3 * W * W, device="cuda")
arena[: 2 * W * W].uniform_(330, 340)
arena[2 * W * W:].uniform_(0, 0.5)
buf = [arena[0:W * W].view(W, W), arena[W * W:2 * W * W].view(W, W)]
pw = arena[2 * W * W:].view(W, W)


def seq(left=False):
    """left: a block at the grid's left edge (window 8704 x 8448, x0 fixed at 0)"""
    cur, s = 0, 0
    for j in range(H // LI):
        m = W - 2 * s
        if left:
            n = W - H - s
            nu.hotspot_leaf(buf[cur][s:s + m, 0:n], pw[s:s + m, 0:n], buf[cur ^ 1][s:s + m, 0:n], LI,
                            gy0=gy + s, gx0=0, rows=R, cols=C)
        else:
            nu.hotspot_leaf(buf[cur][s:s + m, s:s + m], pw[s:s + m, s:s + m], buf[cur ^ 1][s:s + m, s:s + m], LI,
                            gy0=gy + s, gx0=gx + s, rows=R, cols=C)
        cur ^= 1
        s += LI


def fixed():
    cur = 0
    for j in range(H // LI):
        nu.hotspot_leaf(buf[cur], pw, buf[cur ^ 1], LI, gy0=gy, gx0=gx, rows=R, cols=C)
        cur ^= 1


def timed(fn, side=None, n=5):
    fn()
    torch.cuda.synchronize()
    if side:
        side()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(n):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return round(e0.elapsed_time(e1) / n, 3)


hin = torch.empty(1 << 30, dtype=torch.uint8, pin_memory=True)
hout = torch.empty(1 << 30, dtype=torch.uint8, pin_memory=True)
din = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
dout = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def side():
    for _ in range(4):
        with torch.cuda.stream(s1):
            din.copy_(hin, non_blocking=True)
        with torch.cuda.stream(s2):
            hout.copy_(dout, non_blocking=True)


res = {"left_edge_shrinking_ms": timed(lambda: seq(True)), "fixed_ms": timed(fixed), "shrinking_ms": timed(seq), "shrinking_with_copies_ms": timed(seq, side),
       "useful_cells": 8192 * 8192 * H}
res["gcups_shrinking"] = round(res["useful_cells"] / res["shrinking_ms"] / 1e6, 1)
torch.cuda.synchronize()
print(json.dumps(res), flush=True)

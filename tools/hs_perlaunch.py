import json, os, sys
sys.path.insert(0, "/root/repo")
import torch
import paper_conf_ipps_chey19_b200 as nu
W, H, LI = 8704, 256, 8
R = C = 32768
gy, gx = 8192 - H, 8192 - H
arena = torch.empty(3 * W * W, device="cuda")
arena[: 2 * W * W].uniform_(330, 340)
arena[2 * W * W:].uniform_(0, 0.5)
buf = [arena[0:W * W].view(W, W), arena[W * W:2 * W * W].view(W, W)]
pw = arena[2 * W * W:].view(W, W)
def run(kind, reps=5):
    ts = [0.0] * (H // LI)
    for r in range(reps + 1):
        cur, s = 0, 0
        evs = []
        for j in range(H // LI):
            m = W - 2 * s
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            if kind == "left":
                n = W - H - s
                nu.hotspot_leaf(buf[cur][s:s + m, 0:n], pw[s:s + m, 0:n], buf[cur ^ 1][s:s + m, 0:n], LI, gy0=gy + s, gx0=0, rows=R, cols=C)
            elif kind == "left_fixed_w":   # left edge, window width fixed (no column shrink)
                n = W - H
                nu.hotspot_leaf(buf[cur][s:s + m, 0:n], pw[s:s + m, 0:n], buf[cur ^ 1][s:s + m, 0:n], LI, gy0=gy + s, gx0=0, rows=R, cols=C)
            else:
                nu.hotspot_leaf(buf[cur][s:s + m, s:s + m], pw[s:s + m, s:s + m], buf[cur ^ 1][s:s + m, s:s + m], LI, gy0=gy + s, gx0=gx + s, rows=R, cols=C)
            e1.record()
            evs.append((e0, e1))
            cur ^= 1
            s += LI
        torch.cuda.synchronize()
        if r:
            for j, (a, b) in enumerate(evs):
                ts[j] += a.elapsed_time(b) / reps
    return [round(x, 3) for x in ts]
print(json.dumps({k: run(k) for k in ("interior", "left", "left_fixed_w")}))

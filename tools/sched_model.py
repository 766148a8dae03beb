"""Event model of out-of-core schedules (three in-order streams: H2D, compute,
D2H; ops start when their stream is free and their dependencies are done).
Used to compare S2 + drain tail with a wavefront schedule before building it."""
import sys

GiB = 2 ** 30


class Sim:
    def __init__(self, bw_h=49.5e9, bw_d=50.7e9, rate=430e12):
        self.free = {"h": 0.0, "c": 0.0, "d": 0.0}
        self.bw_h, self.bw_d, self.rate = bw_h, bw_d, rate

    def op(self, stream, amount, deps=()):
        dur = amount / (self.bw_h if stream == "h" else self.bw_d if stream == "d" else self.rate)
        t0 = max([self.free[stream]] + list(deps))
        self.free[stream] = t0 + dur
        return t0 + dur

    def end(self):
        return max(self.free.values())


def s2_tail(M, N, K, kc, tail, sr, slots=3, **kw):
    s = Sim(**kw)
    kmain = K - tail
    P = kmain // kc
    leaf_done = [0.0] * P
    a_done, b_done = [], []
    last_c = 0.0
    npieces = tail // kc
    pieces = []
    skip = min(2, max(0, P - 1))
    done_p = 0
    for p in range(P):
        war = leaf_done[p - slots] if p >= slots else 0.0
        a = s.op("h", 4 * M * kc, [war])
        b = s.op("h", 4 * kc * N, [war])
        last_c = s.op("c", 2 * M * N * kc, [a, b, last_c])
        leaf_done[p] = last_c
        while done_p < npieces and p >= skip and (done_p + 1) * (P - skip) <= (p + 1 - skip) * npieces:
            pieces.append(s.op("h", 4 * kc * N)); done_p += 1
    while done_p < npieces:
        pieces.append(s.op("h", 4 * kc * N)); done_p += 1
    bt = max(pieces) if pieces else 0.0
    strip_leaf = []
    r = 0
    while r < M:
        rem = M - r
        rr = sr if rem > 2 * sr else (rem if rem <= 512 else -(-(-(-rem // 2)) // 128) * 128)
        i = len(strip_leaf)
        war = strip_leaf[i - slots] if i >= slots else 0.0
        a = s.op("h", 4 * rr * tail, [war])
        last_c = s.op("c", 2 * rr * N * tail, [a, bt, last_c])
        strip_leaf.append(last_c)
        s.op("d", 4 * rr * N, [last_c])
        r += rr
    return s.end()


def wavefront(M, N, K, kc, S, W, slots=3, **kw):
    """Strip s (M/S rows) processes K panel p at step p + start(s); B panels
    stay resident while some active strip still needs them (window W)."""
    s = Sim(**kw)
    P = K // kc
    sr = M // S
    d = (W - 1) / (S - 1) if S > 1 else 0
    start = [round(i * d) for i in range(S)]
    b_done = [None] * P
    last_c = 0.0
    a_leaf = []            # completion of leaf ops, for A-slot reuse
    steps = P + start[-1]
    for t in range(steps):
        if t < P:
            b_done[t] = s.op("h", 4 * kc * N)
        for i in range(S):
            p = t - start[i]
            if 0 <= p < P:
                war = a_leaf[-slots] if len(a_leaf) >= slots else 0.0
                a = s.op("h", 4 * sr * kc, [war])
                last_c = s.op("c", 2 * sr * N * kc, [a, b_done[p], last_c])
                a_leaf.append(last_c)
                if p == P - 1:
                    s.op("d", 4 * sr * N, [last_c])
    return s.end()


if __name__ == "__main__":
    M = N = K = 32768
    kc = 2048
    for tail in (8192, 12288, 16384, 20480):
        print("S2 tail", tail, round(1e3 * s2_tail(M, N, K, kc, tail, 1920), 1), "ms")
    for S in (8, 16, 32):
        print("wavefront S", S, [(W, round(1e3 * wavefront(M, N, K, kc, S, W), 1)) for W in (1, 4, 8, 12, 16)])

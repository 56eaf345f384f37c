"""Launch-configuration search for the ZVC kernels (§IV-D,
Alg. 1, :170-214; Fig. 5 and Fig. 12 analogues).

Objective: Time_c + Time_dc of one synthetic 500 MB tensor at 50 % sparsity.
The B200 knob: the persistent compress kernel's grid q (1 .. co-resident maximum, SMs x 2) and
its stage/tile variant v (0..9: stages x tile bytes x consumer warps, see cswap.h, which also sets
the block size and the resident CTAs per SM) — cswap_set_zvc_launch.  The decode kernels take one CTA per tile (no free grid parameter).

Searches compared (Fig. 12): Alg. 1 Bayesian optimisation (s1 = 10 random
points, then s2 = 25 points chosen by expected improvement under a Gaussian-process posterior,
written out below with numpy — the paper used fmfn/BayesianOptimization [47], not installed
here), random search with the same 35 evaluations, the "expert" default (q = SMs x 2, v = 0) and
the exhaustive grid (every q x v: Fig. 5's full curve).

    python tools/launch_tune.py [--mb 500] [--s 0.5] [--reps 5] [--out profiles/launch_tune_r02.json]
"""
import argparse
import json
import math
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


class GP:
    """Gaussian-process regression, squared-exponential kernel on inputs scaled to [0,1]^d, targets
    standardised; the length scale is chosen by log marginal likelihood over a small grid."""

    def __init__(self, noise=1e-3):
        self.noise = noise

    def fit(self, X, y):
        import numpy as np
        self.X = np.asarray(X, float)
        y = np.asarray(y, float)
        self.mu, self.sd = y.mean(), y.std() or 1.0
        self.y = (y - self.mu) / self.sd
        best = None
        for ls in (0.05, 0.1, 0.2, 0.4, 0.8):
            K = self._k(self.X, self.X, ls) + self.noise * np.eye(len(self.X))
            L = np.linalg.cholesky(K)
            a = np.linalg.solve(L.T, np.linalg.solve(L, self.y))
            lml = -0.5 * self.y @ a - np.log(np.diag(L)).sum()
            if best is None or lml > best[0]:
                best = (lml, ls, L, a)
        _, self.ls, self.L, self.a = best
        return self

    @staticmethod
    def _k(A, B, ls):
        import numpy as np
        d = ((A[:, None, :] - B[None, :, :]) ** 2).sum(-1)
        return np.exp(-0.5 * d / ls**2)

    def predict(self, Xs):
        import numpy as np
        Ks = self._k(np.asarray(Xs, float), self.X, self.ls)
        m = Ks @ self.a
        v = np.linalg.solve(self.L, Ks.T)
        var = np.clip(1.0 - (v * v).sum(0), 1e-12, None)
        return m * self.sd + self.mu, np.sqrt(var) * self.sd


def expected_improvement(mu, sigma, best, xi=0.01):
    """EI for minimisation."""
    import numpy as np
    z = (best - mu - xi) / sigma
    cdf = 0.5 * (1 + np.vectorize(math.erf)(z / math.sqrt(2)))
    pdf = np.exp(-0.5 * z * z) / math.sqrt(2 * math.pi)
    return (best - mu - xi) * cdf + sigma * pdf


def bayes_opt(space, evaluate, s1=10, s2=25, seed=0):
    """PAPER.md Alg. 1: D <- s1 random points; then s2 times select argmax EI, evaluate, update."""
    import numpy as np
    rng = np.random.default_rng(seed)
    scale = np.array([max(p[i] for p in space) or 1 for i in range(len(space[0]))], float)
    Xall = np.array(space, float) / scale
    D = []
    for i in rng.choice(len(space), size=s1, replace=False):          # lines 3-9
        D.append((space[i], evaluate(space[i])))
    for _ in range(s2):                                                # lines 11-16
        gp = GP().fit(np.array([p for p, _ in D], float) / scale, [y for _, y in D])
        mu, sd = gp.predict(Xall)
        ei = expected_improvement(mu, sd, min(y for _, y in D))
        seen = {p for p, _ in D}
        order = np.argsort(-ei)
        nxt = next(space[i] for i in order if space[i] not in seen)
        D.append((nxt, evaluate(nxt)))
    return min(D, key=lambda t: t[1]), D                              # line 17


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--mb", type=float, default=500)
    ap.add_argument("--s", type=float, default=0.5)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "launch_tune_r01.json"))
    a = ap.parse_args()
    import numpy as np
    import torch

    import synth
    from paper_conf_cluster_chenhzchysc21_b200 import cswap as C
    C.init(0)
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    n = int(a.mb * 1e6) // 4
    x = synth.relu_iid_torch(n, a.s, seed=synth.seed_of(7), dtype=C.F32, device="cuda")
    y = torch.empty_like(x)
    cap = C.max_compressed_size(n, C.F32, C.ZVC)
    buf = torch.empty(cap, dtype=torch.uint8, device="cuda")
    size = torch.zeros(1, dtype=torch.int64, device="cuda")
    err = torch.zeros(1, dtype=torch.int32, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    calls = [0]

    def evaluate(p):
        q, v = p
        C.set_zvc_launch(q, v)
        calls[0] += 1
        ts = []
        for r in range(a.reps + 1):
            flush.fill_(r)
            e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            torch.cuda._sleep(50000)
            e0.record()
            C.compress(x, n, C.F32, C.ZVC, buf, cap, size)
            e1.record()
            C.decompress(buf, cap, y, n, C.F32, C.ZVC, err=err)
            e2.record()
            e2.synchronize()
            if r:
                ts.append(e0.elapsed_time(e2))
        return sorted(ts)[len(ts) // 2]

    grids = list(range(1, 2 * sms + 1))
    NV = 10
    space = [(q, v) for v in range(NV) for q in grids]
    res = {"objective": f"Time_c + Time_dc (ms), ZVC, {a.mb:.0f} MB fp32 at s = {a.s}", "sms": sms}
    t0 = time.time()
    expert = evaluate((0, 0))
    res["expert_default"] = {"q": 2 * sms, "v": 0, "ms": round(expert, 4)}
    t0 = time.time()
    (bp, by), D = bayes_opt(space, evaluate)
    res["bayes_opt"] = {"best": {"q": bp[0], "v": bp[1], "ms": round(by, 4)}, "evaluations": len(D),
                        "seconds": round(time.time() - t0, 2),
                        "trace_ms": [round(min(yy for _, yy in D[:i + 1]), 4) for i in range(len(D))]}
    rng = np.random.default_rng(1)
    t0 = time.time()
    R = [(space[i], evaluate(space[i])) for i in rng.choice(len(space), size=35, replace=False)]
    rp, ry = min(R, key=lambda t: t[1])
    res["random_search"] = {"best": {"q": rp[0], "v": rp[1], "ms": round(ry, 4)}, "evaluations": 35,
                            "seconds": round(time.time() - t0, 2)}
    t0 = time.time()
    full = {p: evaluate(p) for p in space}
    gp_, gy = min(full.items(), key=lambda t: t[1])
    res["grid_search"] = {"best": {"q": gp_[0], "v": gp_[1], "ms": round(gy, 4)}, "evaluations": len(space),
                          "seconds": round(time.time() - t0, 2)}
    res["fig5_curve_ms"] = {f"v{v}": [round(full[(q, v)], 4) for q in grids] for v in range(NV)}
    C.set_zvc_launch(0, -1)
    print(json.dumps({k: v for k, v in res.items() if k != "fig5_curve_ms"}, indent=1))
    with open(a.out, "w") as f:
        json.dump(res, f)


if __name__ == "__main__":
    main()

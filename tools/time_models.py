"""(De)compression time models compared by RAE (SURVEY.md §8(f) NEXT-4a; analogue of PAPER.md
Fig. 10, §V-C :299-303): the paper's piecewise linear regression (LR: one OLS sub-model per
sparsity band on [1, S, S*s], PAPER.md:164-168 — the model libcswap's selector uses) against
Bayesian ridge (BR), support-vector regression (SVM) and a decision tree (DT), all fitted on the
same on-box samples and scored by 5-fold cross-validated RAE = sum|y_hat - y| / sum|mean(y) - y|
(PAPER.md:301).

    python tools/time_models.py --collect 60 --out profiles/time_model_samples_r01.json   (GPU)
    python tools/time_models.py --fit profiles/time_model_samples_r01.json                 (CPU)

Collection: per codec, `--collect` tensors with size uniform in the paper's 20-2000 MB and
sparsity uniform in 20-80 % (the range the paper trains on), iid ReLU-like fp32 (synth), compress and decompress
timed with CUDA events (median of 3 after a warm-up).
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
BANDS = [(0.0, 0.2), (0.2, 0.35), (0.35, 0.5), (0.5, 0.65), (0.65, 0.8), (0.8, 1.01)]


def collect(per_codec: int, out: str, seed: int = 7):
    import numpy as np
    import torch

    import synth
    from paper_conf_cluster_chenhzchysc21_b200 import calibrate, cswap as C
    C.init(0)
    rng = np.random.default_rng(seed)
    maxn = 2000 * 10**6 // 4
    src = torch.empty(maxn, dtype=torch.int32, device="cuda")
    dst = torch.empty_like(src)
    size = torch.zeros(1, dtype=torch.int64, device="cuda")
    err = torch.zeros(1, dtype=torch.int32, device="cuda")
    buf = torch.empty(C.max_compressed_size(maxn, C.F32, C.RLE), dtype=torch.uint8, device="cuda")
    samples = []
    for k in range(per_codec):
        s = float(rng.uniform(0.2, 0.8))
        n = int(rng.uniform(20, 2000) * 10**6) // 4
        src[:n].copy_(synth.relu_iid_torch(n, s, seed=synth.seed_of(6, 0, 0, k), dtype=C.F32, device="cuda"))
        probe = C.probe(src, n, C.F32)
        for codec in (C.ZVC, C.RLE, C.CSR, C.LZ4):
            cap = C.max_compressed_size(n, C.F32, codec)
            tc = calibrate.time_ms(lambda: C.compress(src, n, C.F32, codec, buf, cap, size), 3)
            torch.cuda.synchronize()
            nb = int(size.item())
            tdc = calibrate.time_ms(lambda: C.decompress(buf, nb, dst, n, C.F32, codec, err=err), 3)
            samples.append({"codec": codec, "S": 4 * n, "s": probe.zeros / probe.samples, "true_s": s,
                            "t_c": tc * 1e-3, "t_dc": tdc * 1e-3, "bytes": nb})
        print(f"{k + 1}/{per_codec} S={4 * n / 1e6:.0f}MB s={s:.2f}", flush=True)
    assert int(err.item()) == 0
    with open(out, "w") as f:
        json.dump({"samples": samples, "range": "S 20-2000 MB, s 20-80 %, fp32 iid"}, f)


def rae(pred, y):
    import numpy as np
    pred, y = np.asarray(pred), np.asarray(y)
    return float(np.abs(pred - y).sum() / max(np.abs(y.mean() - y).sum(), 1e-30))


def band_of(s):
    return next(i for i, (a, b) in enumerate(BANDS) if a <= s < b)


class PiecewiseLR:
    """one least-squares sub-model t = b0 + b1*S + b2*S*s per sparsity band."""

    def fit(self, X, y):
        import numpy as np
        self.beta = {}
        bands = np.array([band_of(s) for s in X[:, 1]])
        allb = np.linalg.lstsq(self._A(X), y, rcond=None)[0]
        for b in range(len(BANDS)):
            m = bands == b
            self.beta[b] = np.linalg.lstsq(self._A(X[m]), y[m], rcond=None)[0] if m.sum() >= 3 else allb
        return self

    @staticmethod
    def _A(X):
        import numpy as np
        return np.stack([np.ones(len(X)), X[:, 0], X[:, 0] * X[:, 1]], axis=1)

    def predict(self, X):
        import numpy as np
        return np.array([self._A(x[None])[0] @ self.beta[band_of(x[1])] for x in X])


def models():
    from sklearn.linear_model import BayesianRidge
    from sklearn.pipeline import make_pipeline
    from sklearn.preprocessing import FunctionTransformer, StandardScaler
    from sklearn.svm import SVR
    from sklearn.tree import DecisionTreeRegressor
    feats = FunctionTransformer(lambda X: __import__("numpy").stack([X[:, 0], X[:, 0] * X[:, 1]], axis=1))
    return {
        "LR": PiecewiseLR,
        "BR": lambda: make_pipeline(feats, StandardScaler(), BayesianRidge()),
        "SVM": lambda: make_pipeline(StandardScaler(), SVR(kernel="rbf", C=10.0, epsilon=0.01)),
        "DT": lambda: DecisionTreeRegressor(random_state=0),
    }


def cv_rae(make, X, y, folds=5, seed=0):
    import numpy as np
    idx = np.random.default_rng(seed).permutation(len(y))
    pred = np.empty(len(y))
    for f in range(folds):
        te = idx[f::folds]
        tr = np.setdiff1d(idx, te)
        # targets in ms keep SVR's epsilon meaningful; RAE is scale-free
        pred[te] = make().fit(X[tr], y[tr] * 1e3).predict(X[te]) * 1e-3
    return rae(pred, y)


def fit(path: str) -> dict:
    import numpy as np
    names = {1: "zvc", 2: "rle", 3: "csr", 4: "lz4"}
    d = json.load(open(path))["samples"]
    res = {}
    for codec, nm in names.items():
        pts = [p for p in d if p["codec"] == codec]
        if len(pts) < 10:
            continue
        X = np.array([[p["S"], p["s"]] for p in pts], dtype=float)
        for key in ("t_c", "t_dc"):
            y = np.array([p[key] for p in pts])
            res[f"{nm}_{key[2:]}"] = {m: round(cv_rae(mk, X, y), 4) for m, mk in models().items()}
    mean = {m: round(float(np.mean([r[m] for r in res.values()])), 4) for m in models()}
    return {"per_codec": res, "mean_rae": mean, "samples": len(d), "cv": "5-fold"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--collect", type=int, default=0)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "time_model_samples_r01.json"))
    ap.add_argument("--fit", default=None)
    a = ap.parse_args()
    if a.collect:
        collect(a.collect, a.out)
    if a.fit:
        print(json.dumps(fit(a.fit), indent=1))


if __name__ == "__main__":
    main()

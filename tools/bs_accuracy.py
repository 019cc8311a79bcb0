"""Runs tools/bs_accuracy over market parameters; max element error per variant vs the closed form in
double (scipy erfc), tolerance 1e-5 * max(|ref|, 1) (north_star). Experiment tool, not a test."""
import os, subprocess, sys
import numpy as np
from scipy.special import erfc
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_pldi_dubachcrbf12_b200 import inputs

def exact(S, X, T, r, s):
    S, X, T = (a.astype(np.float64) for a in (S, X, T))
    r, s = float(r), float(s)
    d1 = (np.log(S / X) + (r + s * s / 2) * T) / (s * np.sqrt(T)); d2 = d1 - s * np.sqrt(T)
    N = lambda z: 0.5 * erfc(-z / np.sqrt(2))
    K = X * np.exp(-r * T)
    return S * N(d1) - K * N(d2), K * N(-d2) - S * N(-d1)

n = 1 << 20
S, X, T = inputs.blackscholes_options(n, seed=400)
names = ["lg2S-lg2X, A&S", "lg2(S rcp X), A&S", "lg2S-lg2X, deg7", "lg2(S rcp X), deg7", "deg7 + taylor phi", "ratio + deg7 + taylor phi", "A&S + taylor phi", "ratio + A&S + taylor phi"]
for r, s in [(0.02, 0.30), (0.0, 0.30), (0.10, 0.05), (0.05, 1.0), (0.02, 0.01), (0.0, 0.01), (0.1, 2.0)]:
    r32, s32 = np.float32(r), np.float32(s)
    with open("/tmp/bs_in.bin", "wb") as f:
        f.write(np.array([n], np.int32).tobytes()); f.write(np.array([r32, s32], np.float32).tobytes())
        for a in (S, X, T): f.write(a.tobytes())
    subprocess.run([os.path.join(os.path.dirname(__file__), "bs_accuracy"), "/tmp/bs_in.bin", "/tmp/bs_out.bin"], check=True)
    o = np.fromfile("/tmp/bs_out.bin", np.float32).reshape(8, 2, n)
    C, P = exact(S, X, T, r32, s32)
    row = []
    for v in range(8):
        e = np.maximum(np.abs(o[v, 0] - C) / np.maximum(np.abs(C), 1), np.abs(o[v, 1] - P) / np.maximum(np.abs(P), 1))
        i = int(np.argmax(e))
        row.append("%s: %.3g (S=%.2f X=%.2f T=%.2f)" % (names[v], e[i], S[i], X[i], T[i]))
    print("r=%g sigma=%g | " % (r, s) + " | ".join(row), flush=True)

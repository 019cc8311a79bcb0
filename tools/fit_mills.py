"""Weighted minimax (Lawson) fit of the Mills ratio N(-x)/phi(x) as a polynomial M(k) = sum_{j=1..D} c_j k^j,
k = 1/(1 + p x), minimising max_x phi(x) |M(k) - N(-x)/phi(x)| (the absolute CND error) over x in [0, 40], p scanned.
The map kernel uses D = 7 (p = 0.318): max |dN| = 5.0e-10 (csrc/blackscholes.cu mills7_2)."""
import numpy as np
from scipy.special import erfcx
xx = np.concatenate([np.linspace(0, 10, 20001), np.linspace(10, 40, 3001)])
RR = erfcx(xx/np.sqrt(2))*np.sqrt(np.pi/2); ph = np.exp(-xx*xx/2)/np.sqrt(2*np.pi)
def lawson(p, D, it=300):
    k = 1/(1+p*xx); V = np.stack([k**j for j in range(1, D+1)], 1)
    A = ph[:,None]*V; b = ph*RR
    u = np.ones(len(xx))/len(xx)
    for _ in range(it):
        sw = np.sqrt(u)
        co = np.linalg.lstsq(A*sw[:,None], b*sw, rcond=None)[0]
        r = np.abs(A@co - b)
        u = u*r; u /= u.sum()
    return co, np.max(np.abs(A@co-b))
import sys
for D in [int(a) for a in sys.argv[1:]] or (5, 6, 7, 8):
    best=None
    for p in np.linspace(0.15, 0.7, 23):
        co,e = lawson(p,D,100)
        if best is None or e<best[2]: best=(p,co,e)
    p0=best[0]
    for p in np.linspace(p0-0.025, p0+0.025, 26):
        co,e = lawson(p,D,300)
        if e<best[2]: best=(p,co,e)
    p,co,e=best
    print(D, "p=%.6f"%p, "max|dN|=%.3g"%e, "coef", ", ".join("%.10e"%c for c in co))

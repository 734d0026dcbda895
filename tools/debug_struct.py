import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_sc_0007k13_b200 import inputs, siac
k = int(sys.argv[1]) if len(sys.argv) > 1 else 1
N = 16
V, T = inputs.structured_mesh(N)
C = inputs.random_modes(len(T), k, seed=k)
h = 1.0 / N
g1 = np.arange(0, N + 1) / N
g2 = (np.arange(0, N) + 0.5) / N
X = np.concatenate([g1, g2])
P = np.array([[x, y] for x in X[::3] for y in X[::2]])
ctx = siac.create(V, T, C, k, h)
ctx.set_schedule(2); a = ctx.eval(P)
ctx.set_schedule(4); b = ctx.eval(P)
d = np.abs(a - b)
print("variant", os.environ.get("SIAC_LIB_VARIANT"), "k", k, "max diff", d.max())
for i in np.argsort(-d)[:5]:
    print(i, P[i], a[i], b[i], d[i])

"""Debug: runs one SDDMM problem through a VS_TC_TRACE build of libvs (VS_LIB_PATH) and prints
CTA 0's pipeline timeline (producer stage issue, MMA full-wait done, epilogue tile ready)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_sc_chenqldx21_b200 as vs
from synth import gen
M, K, N, V, S = [float(x) if i == 4 else int(x) for i, x in enumerate(sys.argv[1:6])]
rng = gen.make_rng("trace")
W = torch.from_numpy(gen.colvec_dense(rng, M, K, V, 1 - S)).cuda()
X = torch.from_numpy(gen.dense_operand(rng, K, N)).cuda()
G = torch.from_numpy(gen.dense_operand(rng, M, N)).cuda()
rp, ci, va = vs.encode(V, dense=W)
for _ in range(3):
    out = vs.sddmm(rp, ci, G, X, V)
torch.cuda.synchronize()
buf = (ctypes.c_ulonglong * (3 * 4096))()
print("rc", vs.load().vs_debug_tc_trace(buf))
a = np.frombuffer(buf, dtype=np.uint64).reshape(3, 4096).astype(np.int64)
t0 = a[0][0]
for role, name in enumerate(["produced", "mma_full", "epi_tile"]):
    r = a[role]; n = int((r > 0).sum())
    print(name, n, (r[:min(n, 48)] - t0).tolist())

import sys, numpy as np
sys.path.insert(0, '/root/repo'); sys.path.insert(0, '/root/repo/tests')
import torch, synth, oracle
import paper_conf_ipps_gatesklpd17_b200 as bsp
n, batch = 20, 8192 + 77
b = np.arange(batch, dtype=np.uint64)
canon = synth.generate(n, "als", 5, b, upper="mirror", fail_seed=6, fail_period=31)
dA = torch.from_numpy(canon.reshape(-1).copy()).cuda()
di = torch.zeros(batch, dtype=torch.int32, device="cuda")
bsp.batch_spotrf_canonical(n, batch, dA, di)
src = torch.from_numpy(canon.reshape(-1).copy()).cuda()
inter = torch.zeros(bsp.batch_interleaved_elems(n, batch, 32), device="cuda")
bsp.batch_canonical_to_interleaved(n, batch, 32, src, inter)
d2 = torch.zeros(batch, dtype=torch.int32, device="cuda")
bsp.batch_spotrf_interleaved(n, batch, 32, inter, d2)
torch.cuda.synchronize()
i1, i2 = di.cpu().numpy(), d2.cpu().numpy()
L64, i64 = oracle.potrf(n, canon)
bad = np.nonzero(i1 != i2)[0]
print("mismatch", bad.size, "canon-vs-oracle", int((i1 != i64).sum()), "inter-vs-oracle", int((i2 != i64).sum()))
for k in bad[:10]: print(k, i1[k], i2[k], i64[k])
print(bsp.bspotrf_get_tuning(n, 32).as_dict())

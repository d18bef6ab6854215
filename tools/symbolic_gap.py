import sys, torch, numpy as np
sys.path.insert(0, ".")
import paper_conf_ipps_ramamoorthybsk15_b200 as spg, workloads as W
A, _ = W.make("webbase1m")
dA = spg.DeviceCSR.from_host(A, "cuda:0")
h = spg.spg_create(0, None, torch.float64)
spg.spg_set_option(h, "timing", 1)
rp = torch.empty(A.nrows + 1, dtype=torch.int64, device="cuda:0")
nnz, rb, re = spg.spg_spgemm_symbolic(h, dA, dA, rp)
col = torch.empty(nnz, dtype=torch.int32, device="cuda:0"); val = torch.empty(nnz, dtype=torch.float64, device="cuda:0")
spg.spg_spgemm_numeric(h, dA, dA, rp, col, val)
torch.cuda.synchronize()
st = torch.cuda.current_stream()
res = []
for k in range(20):
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True); e2 = torch.cuda.Event(enable_timing=True)
    e0.record(st); spg.spg_spgemm_symbolic(h, dA, dA, rp); e1.record(st); spg.spg_spgemm_numeric(h, dA, dA, rp, col, val); e2.record(st)
    torch.cuda.synchronize()
    s = spg.spg_get_stats(h)
    res.append((e0.elapsed_time(e1), s["ms_analysis"], s["ms_symbolic"], e1.elapsed_time(e2), s["ms_numeric"]))
r = np.median(np.array(res), axis=0)
print("sym_call %.4f  analysis %.4f  symbolic_kernels %.4f  -> post-scan overhead %.4f ms; num_call %.4f num_events %.4f" % (r[0], r[1], r[2], r[0]-r[1]-r[2], r[3], r[4]))

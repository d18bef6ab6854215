# compute-sanitizer passes on small inputs (memcheck: out-of-bounds / misaligned; racecheck and
# synccheck: shared-memory hazards and barrier misuse in the block-cooperative kernels)
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
cat > /tmp/san_case.py <<'PY'
import sys, torch, numpy as np
sys.path.insert(0, ".")
import paper_conf_ipps_ramamoorthybsk15_b200 as spg, workloads as W
A, _ = W.make("cl10k")
dA = spg.DeviceCSR.from_host(A, "cuda:0")
for opts in ({}, {"force_class": 6}, {"force_class": 5}, {"light_max_flops": 0}, {"light_max_flops": 4096, "tile_flops": 1024},
             {"heavy_sort": 1}, {"pack_b": 1}, {"heavy_order": 2}):
    plan = spg.SpGEMM(0, torch.float64)
    for k, v in opts.items():
        plan.set_option(k, v)
    C = plan(dA, dA)
    torch.cuda.synchronize()
    plan.close()
D = torch.rand(A.ncols, 40, dtype=torch.float64, device="cuda:0")
spg.csrmm(dA, D, csrmm_light_nnz=16)
B = W.random_csr(A.ncols, 3000, 0.002, 4, canonical=False)
dB = spg.DeviceCSR.from_host(B, "cuda:0")
plan = spg.SpGEMM(0, torch.float64, input_canonical=0)
C2 = plan(dA, dB)
torch.cuda.synchronize()
plan.close()
print("case ok", int(C.row_ptr[-1]), int(C2.row_ptr[-1]))
PY
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 python /tmp/san_case.py > gpurun_out/san_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|case ok" gpurun_out/san_$tool.log | tail -3
done

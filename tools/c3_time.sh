timeout 600 python -c "
import sys, torch; sys.path.insert(0,'.')
import paper_conf_ipps_metzgd23_b200 as dt
X, y = dt.dt_gen_table(3, 100_000_000, d=32, cnn_pool_bits=22, gpu_pool_bits=12, device='cuda')
t = dt.dt_fit(X, y, 16, 1); torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(3): t = dt.dt_fit(X, y, 16, 1)
b.record(); torch.cuda.synchronize()
print('c3 ms/fit', a.elapsed_time(b)/3, t.size)
dt.dt_release_workspace()
dt.dt_profile_reset(); dt.dt_profile_enable(True); dt.dt_fit(X, y, 16, 1); dt.dt_profile_enable(False)
print({k: round(v['ms'],1) for k, v in dt.dt_profile().items() if v['ms'] > 1})
"

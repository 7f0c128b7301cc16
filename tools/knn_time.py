import sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_metzgd23_b200 as dt
X, y = dt.dt_gen_table(1, 1 << 16, d=16, device="cuda")
Xq, _ = dt.dt_gen_table(2, 1 << 20, d=16, device="cuda")
out = dt.dt_knn_predict(X, y, Xq[:4096], 5)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record(); o = dt.dt_knn_predict(X, y, Xq, 5); b.record(); torch.cuda.synchronize()
print(sys.argv[1], a.elapsed_time(b), float(o.sum()))

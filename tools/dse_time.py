"""Times dt_predict_dse on the bench's configs[3] shape (measurement helper)."""
import sys

import torch

sys.path.insert(0, '.')
import datagen  # noqa: E402
import paper_conf_ipps_metzgd23_b200 as dt  # noqa: E402

X, y = dt.dt_gen_table(1, 1_000_000, d=16, device="cuda")
tree = dt.dt_fit(X, y, 20, 128)
cnn, gpu, src = datagen.dse_tables(3, 0, 1 << 20, 1 << 10)
cd, gd = torch.from_numpy(cnn).cuda(), torch.from_numpy(gpu).cuda()
out = torch.empty((1 << 30), dtype=torch.float64, device="cuda")
for _ in range(2):
    dt.dt_predict_dse(tree, cd, gd, src, out=out)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(3):
    dt.dt_predict_dse(tree, cd, gd, src, out=out)
b.record()
torch.cuda.synchronize()
ms = a.elapsed_time(b) / 3
print(sys.argv[1] if len(sys.argv) > 1 else "", f"{ms:.2f} ms/pass, {(1 << 30) / ms / 1e6:.1f} G preds/s", float(out[:1 << 20].sum()))

"""Pack-walk microbench on the C2 cut-0 live set (535 tensors, 205 MB), CUDA events."""
import os, sys, torch
sys.path.insert(0, ".")
from paper_conf_middleware_wur0hdh21_b200 import ops as K
from sf_inputs import graphs as G
g = G.resnet50_forest(batch=1)
sizes = [t.nbytes for t in g.tensors if t.kind in (0, 1, 2)]
ru = lambda x, a: (x + a - 1) // a * a
src = torch.empty(sum(ru(s, 256) for s in sizes), dtype=torch.uint8, device="cuda")
dst = torch.empty_like(src)
descs, so = [], 0
for s_ in sizes:
    descs.append((src.data_ptr() + so, dst.data_ptr() + so, s_, ru(s_, 256))); so += ru(s_, 256)
tot = sum(sizes)
for _ in range(3): K.mtcopy(descs)
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
ts = []
for _ in range(10):
    e0.record(); K.mtcopy(descs); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
t = sorted(ts)[len(ts) // 2] * 1e-3
x = torch.empty(tot // 4, device="cuda"); y = torch.empty_like(x)
e0.record(); y.copy_(x); e1.record(); torch.cuda.synchronize()
for _ in range(5): y.copy_(x)
e0.record(); y.copy_(x); e1.record(); torch.cuda.synchronize()
tc = e0.elapsed_time(e1) * 1e-3
print(f"BPS={os.environ.get('SF_COPY_BPS','8')} MIN={os.environ.get('SF_COPY_MINCHUNKS','2048')}: "
      f"pack {2*tot/t/1e9:.0f} GB/s ({t*1e6:.1f} us)   torch copy same bytes {2*tot/tc/1e9:.0f} GB/s")

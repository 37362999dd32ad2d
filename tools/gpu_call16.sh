python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo build=$?
timeout 900 python -m pytest tests/test_gpu_place.py tests/test_gpu_topk.py -q -x 2>&1 | tail -3
timeout 300 python -c "
import sys, time, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import synth
g = synth.generate('C4'); G = insta.Graph(g)
G.forward(3.0, 0.0); d = G.backward(); w = -(d[:, 0] + d[:, 1])
x = torch.rand(g.num_pins, device='cuda') * 1000; y = torch.rand(g.num_pins, device='cuda') * 1000
for _ in range(3): G.timing_loss(x, y, w, 1e-3)
torch.cuda.synchronize(); e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(10): G.timing_loss(x, y, w, 1e-3)
e1.record(); torch.cuda.synchronize(); print('C4 timing_loss ms', e0.elapsed_time(e1) / 10)
"

"""Diagnostic: per-layer forward drift of the ResNet-101 b32 training graph vs the fp64 oracle
(rel L2 of every ReLU input), to see whether drift grows with depth or jumps at one layer."""
import copy
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import torch  # noqa: E402
from oracle import model as om  # noqa: E402
from synth import inputs as si  # noqa: E402
from paper_conf_eurosys_stratimk24_b200 import workloads as W, collocate as C  # noqa: E402
import parity as PT  # noqa: E402

torch.cuda.set_device(0)
layers = W.RESNET101_LAYERS if (len(sys.argv) < 2 or sys.argv[1] == "101") else W.RESNET50_LAYERS
b = int(sys.argv[2]) if len(sys.argv) > 2 else 32
P = si.make_params(W.resnet_train_spec(layers))
xs = [si.normal((b, 224, 224, 3), si.HP_SEED, sub=0)]
labs = [si.labels(b, 1000, si.HP_SEED, sub=0)]
g = W.resnet_train_graph(P, xs, labs, layers=layers)
be = C.BEClient(g)
g.params.reset()
C.run_session(be=be, be_iters=1)
masks = {k: v.cpu() for k, v in g.relu_in.items()}
tr = {}
loss, newP, _, grads = om.resnet_train_step(P, {}, xs[0], labs[0], first=True, layers=layers, masks=masks, trace=tr)
print("loss rel", PT.rel(g.loss, loss.reshape(1)))
order = ["bn1"] + [k for k in tr["relu_in"] if k != "bn1"][::-1]
for k in order:
    o = tr["relu_in"][k]
    print(f"{k:16s} rel {PT.rel(masks[k], o):.3e} elem {PT.elem(masks[k], o):.3e}")

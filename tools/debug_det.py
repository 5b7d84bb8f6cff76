import sys, os
sys.path[:0] = [os.path.join(os.path.dirname(__file__), '..')]
import torch
from synth import inputs as si
import paper_conf_eurosys_stratimk24_b200 as orion
from paper_conf_eurosys_stratimk24_b200 import workloads as W
b, hw = int(sys.argv[1]), int(sys.argv[2])
P = si.make_params(W.mnv2_spec())
g = W.mnv2_train_graph(P, [si.normal((b, hw, hw, 3), si.BE_SEED, sub=0)], [si.labels(b, 1000, si.BE_SEED, sub=0)])
s = torch.cuda.current_stream().cuda_stream
snap = None
for rep in range(3):
    g.params.reset()
    outs = []
    for i, (fn, args, lab) in enumerate(g.ops):
        orion.kernel_launch(fn, args, s)
        torch.cuda.synchronize()
        # checksum the op's output buffer (arg index by fn)
        outs.append(lab)
    print("rep", rep, "loss", float(g.loss), "gsum", float(g.params.gflat.double().sum()))

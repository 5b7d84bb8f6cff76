import sys, os
sys.path[:0] = [os.path.join(os.path.dirname(__file__), '..'), os.path.join(os.path.dirname(__file__), '..', 'tests')]
import torch
from synth import inputs as si
from oracle import model as om
import paper_conf_eurosys_stratimk24_b200 as orion
from paper_conf_eurosys_stratimk24_b200 import workloads as W, collocate as C
b, hw = int(sys.argv[1]), int(sys.argv[2])
P = si.make_params(W.mnv2_spec())
xs = [si.normal((b, hw, hw, 3), si.BE_SEED, sub=0)]
labels = [si.labels(b, 1000, si.BE_SEED, sub=0)]
g = W.mnv2_train_graph(P, xs, labels)
s = torch.cuda.current_stream().cuda_stream
for fn, args, lab in g.ops:
    orion.kernel_launch(fn, args, s)
torch.cuda.synchronize()
l_direct = float(g.loss)
g.params.reset()
be = C.BEClient(g)
C.run_session(be=be, be_iters=1)
l_sched = float(g.loss)
loss_ref, newP, newV, g_ref = om.mnv2_train_step(P, {}, xs[0], labels[0], first=True)
print("b", b, "hw", hw, "direct", l_direct, "sched", l_sched, "oracle", float(loss_ref))
logits = g.logits.cpu()
print("logit norm", float(logits.norm()))

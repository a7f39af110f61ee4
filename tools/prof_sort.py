"""Small driver for ncu: a few device sorts of n uniform float64 keys (default 2^28)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import hsort_inputs  # noqa: E402
import paper_conf_ipps_gowanlockk18a_b200 as hs  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 28
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
hs.hsort_init()
A = hsort_inputs.generate("uniform", n, seed=2)
d_in = torch.from_numpy(A).cuda()
d_out = torch.empty_like(d_in)
for _ in range(reps):
    hs.hsort_sort_device(d_in, d_out)
torch.cuda.synchronize()
print("done", n, reps)
hs.hsort_finalize()

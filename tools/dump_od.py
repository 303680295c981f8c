"""Write the out-degrees d~ (original ids) of a config's graph as raw u32 (for
tools/aorder_bench.cpp):  python tools/dump_od.py CFG DIRECT OUT"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen  # noqa: E402
import paper_conf_sigmod_hu0l21_b200 as tc  # noqa: E402

cfg, d, out = int(sys.argv[1]), sys.argv[2], sys.argv[3]
spec = graphgen.CONFIGS[cfg]
src = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
dst = torch.empty(spec.samples, dtype=torch.int32, device="cuda")
graphgen.generate_cuda(spec, src.data_ptr(), dst.data_ptr(), torch.cuda.current_stream().cuda_stream)
torch.cuda.synchronize()
g = tc.Graph(src, dst, spec.n).direct(d)
g.export_direct().tofile(out)
g.free()

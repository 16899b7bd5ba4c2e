import os, sys, time
sys.path.insert(0, '.')
os.environ['SG_DEBUG_MEM'] = '1'
import torch
from paper_conf_ipps_wuk13_b200 import binding as B
from synth import graphs as SG
torch.cuda.set_device(0)
g = SG.make('gos2m', cache=False)
for it in range(3):
    h = B.shingle_graph_create(g.row_ptr, g.col)
    t = time.time()
    B.shingle_pass(h, 2, 200, 201); B.group_by_shingle(h); B.shingle_pass(h, 2, 200, 202); B.group_by_shingle(h)
    print('step', it, time.time() - t, B.sg_get_stage_ms(h), file=sys.stderr, flush=True)
    B.shingle_graph_destroy(h)
    print('after destroy', torch.cuda.mem_get_info(), file=sys.stderr, flush=True)

"""Diagnose test_pool_growth_retry_with_length_groups: run variants with stats."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, readgen
import paper_conf_ipps_goswamilsp18_b200 as lz
variant = sys.argv[1]
lpp = int(sys.argv[2])
for kv in variant.split(","):
    if "=" in kv:
        k, v = kv.split("=")
        os.environ[k] = v
reads = readgen.reads(7, 20_000, 3000, 64, 0.01)
packed = lz.load_reads(torch.from_numpy(reads).cuda())
t = time.time()
r = lz.greedy_graph(packed, 3000, 64, 1, lengths_per_pass=lpp)
torch.cuda.synchronize()
print(variant, lpp, "%.2fs" % (time.time() - t), r.stats, flush=True)

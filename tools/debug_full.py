import sys, os, math
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_junger0s18_b200 as wd, wdgen
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests")); from wdtest import to_dev
for n in (300001, 1 << 20):
  for alpha in (0.95, 0.99, 0.999):
    for K in (4, 8):
      for G in (1, 4, 32):
        keys, vals = wdgen.unique_keys(n, 7), wdgen.values(n, 8)
        t = wd.Table(int(math.ceil(n / alpha)), 1, G)
        t.set_option(wd.WD_OPT_KEYS_IN_FLIGHT, K)
        t.insert(to_dev(keys), to_dev(vals)); torch.cuda.synchronize()
        st = t.sync(); c = t.counters(); sl = t.dump()
        k = (sl & np.uint64(0xFFFFFFFF)).astype(np.uint32); k = k[k != np.uint32(0xFFFFFFFF)]
        u, cnt = np.unique(k, return_counts=True)
        missing = np.setdiff1d(keys, u).size
        print(f"n={n} a={alpha} K={K} G={G} st={st} {c} occupied={k.size} dups={(cnt>1).sum()} missing={missing}", flush=True)
        t.close()

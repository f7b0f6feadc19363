import sys, os, math
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R); sys.path.insert(0, os.path.join(R, "tests"))
import numpy as np, torch
import paper_conf_ipps_junger0s18_b200 as wd, wdgen, oracle
from wdtest import to_dev
n = 300001
for trial in range(int(os.environ.get('TRIALS', '40'))):
  for alpha in (0.999,):
    for K in (4, 8):
      for G in (4,):
        keys, vals = wdgen.unique_keys(n, 7 + trial), wdgen.values(n, 8)
        t = wd.Table(int(math.ceil(n / alpha)), 1, G)
        t.set_option(wd.WD_OPT_KEYS_IN_FLIGHT, K)
        t.insert(to_dev(keys), to_dev(vals)); torch.cuda.synchronize()
        st = t.sync(); c = t.counters(); sl = t.dump(); cap = t.capacity()
        k = (sl & np.uint64(0xFFFFFFFF)).astype(np.uint32)
        if st or trial < 2: print(f"trial={trial} a={alpha} K={K} G={G} st={st} {c} cap={cap} empty={int((k==0xFFFFFFFF).sum())}", flush=True)
        if c["failed"]:
            fk = c["last_failed_key"]
            full = 0
            for p in range(1024):
                b = oracle.Replay.base(fk, p, cap)
                full += int(np.all(k[b:b+32] != 0xFFFFFFFF))
            print("   failed key", hex(fk), "in table:", bool(np.any(k == fk)), "full regions of its 1024:", full, flush=True)
        t.close()

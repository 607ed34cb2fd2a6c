import sys, threading, numpy as np
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
import gen, oracle, wjformat, paper_conf_ipps_weij11_b200 as wj
from test_gpu_multi import dist_index
text, off = gen.generate(gen.CONFIGS[1])
want = wjformat.parse(oracle.index_bytes(text, off))
slices, _ = dist_index(text, off, 2, cuts=[0, 400, 1000])
got = wjformat.parse(wj.merge_serialized(slices))
for h in ["n_docs", "n_tokens", "n_dropped", "n_terms", "n_postings", "n_term_bytes"]:
    print(h, getattr(got, h), getattr(want, h))
gd, wd = got.as_dict(), want.as_dict()
bad = [t for t in wd if gd.get(t) != wd[t]]
print("bad terms", len(bad), "of", len(wd))
for t in bad[:5]:
    print(t, wd[t][:6], gd.get(t, [])[:6])
a = wj.merge_serialized(slices); b = oracle.index_bytes(text, off)
i = next((k for k in range(min(len(a), len(b))) if a[k] != b[k]), None)
print("len", len(a), len(b), "first diff", i)
print("cf equal", np.array_equal(got.cf, want.cf), "df equal", np.array_equal(got.df, want.df))
for r, sl in enumerate(slices):
    x = wjformat.parse(sl)
    print("slice", r, x.n_tokens, int(x.cf.sum()), int(x.tf.sum()))

import numpy as np, torch, sys
sys.path.insert(0, '.')
import harmonia_gen as gen, paper_conf_ppopp_yanlpz19_b200 as hm
keys = gen.uniform_keys(1 << 16); vals = gen.values_for(keys)
t = hm.Tree(torch.from_numpy(keys).cuda(), torch.from_numpy(vals).cuda(), fanout=16)
q = torch.from_numpy(gen.uniform_queries(keys, 1 << 20)).cuda()
out = t.search(q); torch.cuda.synchronize()
print("ok", np.array_equal(out.cpu().numpy(), gen.values_for(q.cpu().numpy())))

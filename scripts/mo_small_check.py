import sys, os
sys.path.insert(0, os.getcwd())
import torch, numpy as np, ragen, oracle
import paper_conf_ipps_wudwcyc12_b200 as R
for n in (3*8192+5, (1<<21)+77):
    x = ragen.int32_column(2, n)
    xd = torch.from_numpy(x).cuda()
    ch = [[("lt", 0)]]
    outs, cnts = R.select_multi(xd, ch)
    torch.cuda.synchronize()
    e = oracle.select_multi(x, ch)[0]
    print(n, int(cnts[0]), e.size, np.array_equal(outs[0][:e.size].cpu().numpy(), e), flush=True)

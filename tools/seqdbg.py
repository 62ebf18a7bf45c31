import sys; sys.path.insert(0,'.')
import numpy as np, torch
from fsmgen import dfas, streams
from oracle import seq
from paper_conf_ppopp_xiaja20_b200 import fsmspec
from paper_conf_ppopp_xiaja20_b200.fsmspec import FSM
d = dfas.random_dfa(16, 5, seed=9)
data = streams.splitmix_bytes(9, 0, 200_017)
x = torch.from_numpy(data.copy()).cuda()
f = FSM.from_dfa(d); f.set_options(merge=1)
print(f.run_spec_k(x.data_ptr(), data.size, 1), seq.run(d, data))

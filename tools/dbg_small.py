import sys; sys.path.insert(0,'.')
import numpy as np
import paper_conf_icpp_yasudonitkyi20_b200 as P
from workloads import random_qubo
for n,S in [(16,4),(100,3),(1024,2),(1100,2),(3000,2),(5000,2),(10000,2)]:
    try:
        s=P.Solver(random_qubo(n,1), searches=S, local_flips=50, pool_size=4, seed=1)
        s.search(2); print(n,'ok',s.round_results()[1]); s.close()
    except Exception as e: print(n,'ERR',e); break

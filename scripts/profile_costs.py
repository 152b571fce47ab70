import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_cluster_ajipbf15_b200 import Mapper, workloads
E, Q, D = (int(v) for v in sys.argv[1:4]) if len(sys.argv) > 3 else (100_000, 8, 4)
model = workloads.cost_model(42, E, Q, D)
dm = {k: (torch.from_numpy(np.ascontiguousarray(v)).cuda() if isinstance(v, np.ndarray) else v) for k, v in model.items()}
with Mapper(0) as m:
    for _ in range(3):
        m.build_costs(dm, D, device_out=True)
    torch.cuda.synchronize()

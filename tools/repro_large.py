"""Repro helper: one irr_getrf call on a few large G1 matrices (few-large regime)."""
import sys
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import irrgen
from paper_conf_sc_abdelfattahgbtld22_b200 import irr
from paper_conf_sc_abdelfattahgbtld22_b200.batch import MatrixBatch

shapes = [tuple(int(x) for x in s.split("x")) for s in sys.argv[1:]] or [(8192, 700)]
B = MatrixBatch([s[0] for s in shapes], [s[1] for s in shapes])
host = np.zeros(B.total)
for i, (m, n) in enumerate(shapes):
    B.matrix(i, host)[:, :] = irrgen.uniform_values(1, i, m, n)
B.data.copy_(torch.from_numpy(host))
B.getrf()
torch.cuda.synchronize()
print("ok", B.info.cpu().numpy()[: B.batch])

"""Dev helper: repeat spmv_exec and report rows whose bits change between runs."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_ispass_balajicjk23_b200 import spmv  # noqa: E402
from oracle import plan as oplan  # noqa: E402

dev = torch.device("cuda:0")
for cfg in (4, 2, 1):
    A = synth.config(cfg, small=True).A
    perm, _ = spmv.reorder(A.row_ptr, A.col, "rabbit")
    for win in (True, False):
        P = spmv.Plan(torch.from_numpy(A.row_ptr).to(dev), torch.from_numpy(A.col).to(dev),
                      torch.from_numpy(A.val).to(dev), torch.from_numpy(perm).to(dev),
                      smem_window=win)
        x = torch.from_numpy(synth.vector(A.n, 3)).to(dev)
        xB = P.permute_vec(x)
        ys = [P.exec(xB).cpu().numpy().view(np.int32).copy() for _ in range(20)]
        bad = set()
        for y in ys[1:]:
            bad |= set(np.nonzero(y != ys[0])[0].tolist())
        tiles = P.export_bins()["tiles"].cpu().numpy()
        info = P.info()
        bt = sorted({int(np.searchsorted(tiles, r, side="right") - 1) for r in bad})
        print(f"cfg{cfg} win={win} n={A.n} tiles={info['n_tiles']} bad_rows={len(bad)} "
              f"bad_tiles={bt[:20]}", flush=True)
        P.close()

"""Calibrate the integer roof on the box: IMAD/clk/SM (independent mad.lo chains)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_lucw0cz25_b200 import bzk
import torch
torch.cuda.init()
r = [bzk.bzk_debug_imad_rate(1 << 14) for _ in range(3)]
print(json.dumps({"imad_per_clk_per_sm": r}))

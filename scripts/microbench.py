"""Calibrate the integer roof on the box: IMAD, IMAD.WIDE and Montgomery-product rates per SM per clock."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_lucw0cz25_b200 import bzk
import torch
torch.cuda.init()
names = {0: "imad_per_clk_sm", 1: "imad_wide_per_clk_sm", 2: "mont_mul_v1_per_clk_sm", 3: "mont_mul_per_clk_sm", 4: "dfma_per_clk_sm", 5: "mont_mul_1chain_16warps", 6: "mont_mul_2chain_16warps",
         7: "mont_mul_4chain_16warps", 8: "mont_mul2_per_clk_sm",
         9: "fp64_mont_mul2_per_clk_sm", 10: "mixed_warps_int_fp64_mont_mul2_per_clk_sm",
         11: "mixed_in_thread_int_fp64_mont_mul2_per_clk_sm"}
out = {names[k]: round(bzk.bzk_debug_bench(k, 1 << 12 if k in (0, 1, 4) else 1 << 9), 4) for k in names}
out["mont_mul_imad_slots"] = round(out["imad_per_clk_sm"] / out["mont_mul_per_clk_sm"], 1)
print(json.dumps(out))

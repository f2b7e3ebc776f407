"""Where does the fault-free FT2-on run clip?  Per critical layer (name,
block) of the C5 campaign model: the share of (row, decode step) outputs with
a correction, and the decode/prefill magnitude ratio."""
import os, sys, json
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
from paper_conf_hpdc_sunzmg00y25_b200.runner import CONFIGS, Runner
from paper_conf_hpdc_sunzmg00y25_b200 import campaign

model = sys.argv[1] if len(sys.argv) > 1 else "llama-2-7b"
B, T, S = int(os.environ.get("B", "256")), 16, 32
r = Runner(CONFIGS[model], B, T, S + 1, seed=1, device="cuda", outliers=os.environ.get("OUTLIERS", "1") == "1")
p = campaign.campaign_prompts(r)
g = campaign.golden_runs(r, p)
corr = r.state.corrected.view(r.cfg.n_layers, len(r.crit_names), B)
out = {"model": model, "rows_with_any_correction": float((corr.sum((0, 1)) > 0).float().mean()),
       "fault_free_token_mismatch": float((g.tok_on != g.tok_off).any(1).float().mean())}
per = {}
for j, n in enumerate(r.crit_names):
    c = corr[:, j, :]
    per[n] = {"rows_corrected_share": float((c > 0).float().mean()), "neurons_per_row": float(c.float().mean()),
              "by_block_rows_share": [round(float((c[b] > 0).float().mean()), 3) for b in range(r.cfg.n_layers)]}
out["per_layer"] = per
b = r.state.bounds.float().view(r.cfg.n_layers, len(r.crit_names), B, 2)
out["bounds_hi_median_by_layer"] = {n: [round(float(b[k, j, :, 1].median()), 3) for k in range(0, r.cfg.n_layers, 4)]
                                    for j, n in enumerate(r.crit_names)}
print(json.dumps(out))

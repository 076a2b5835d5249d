"""cfg5 records leg of bench.py at several worker counts (usage: cfg5_workers.py 1:0,8:32 -- workers:min windows per warp)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

for wm in (sys.argv[1] if len(sys.argv) > 1 else "8:32").split(","):
    w, m = (int(x) for x in wm.split(":"))
    r = bench.measure_cfg5_records(ve, torch.cuda.current_stream(), 6539.9, workers=w, min_wpw=m)
    print(json.dumps({k: r[k] for k in ("workers", "min_windows_per_warp", "ms", "records_per_s", "analyze_ms_this_rank_sum_over_workers",
                                        "closed_forms_ok", "closed_forms_kernels_checked")}), flush=True)

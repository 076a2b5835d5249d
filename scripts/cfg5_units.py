"""cfg5 records leg in units mode at several batch sizes / worker counts (usage: cfg5_units.py 500:2,1000:1)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_asplos_zhouhmm022_b200 import ve  # noqa: E402

for bw in (sys.argv[1] if len(sys.argv) > 1 else "500:2").split(","):
    b, w = (int(x) for x in bw.split(":"))
    r = bench.measure_cfg5_units(ve, torch.cuda.current_stream(), 6539.9, batch=b, workers=w)
    print(json.dumps({k: r[k] for k in ("mode", "batches", "ms", "records_per_s", "closed_forms_ok",
                                        "closed_forms_kernels_checked", "closed_form_mismatches")}), flush=True)

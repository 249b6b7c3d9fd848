"""kf_run_host_async over a stream of C3 images: ms per image for several
band counts (option host_bands).  Diagnostics only."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from kf_inputs import gen  # noqa: E402
from kf_inputs import pipelines as P  # noqa: E402
from paper_conf_cgo_qiaorht19_b200 import kfuse as K  # noqa: E402

spec, seed = P.config(sys.argv[1] if len(sys.argv) > 1 else "C3")
W, H = spec["width"], spec["height"]
host = gen.image(spec["dtype"], seed, W, H)
hin = torch.from_numpy(host).pin_memory()
hout = torch.empty_like(hin).pin_memory()
st = torch.cuda.Stream()
for nb in (1, 2, 3, 4, 6, 8, 12):
    for asyn in (True, False):
        plan = K.Pipeline.from_spec(spec, {"host_bands": nb}).plan_fusion("b200")
        run = plan.run_host_async if asyn else plan.run_host
        for _ in range(3):
            run([hin], [hout], st)
        st.synchronize()
        res = []
        for _ in range(5):
            t = time.perf_counter()
            for _ in range(20):
                run([hin], [hout], st)
            st.synchronize()
            res.append((time.perf_counter() - t) / 20 * 1e3)
        res.sort()
        print(json.dumps({"cfg": spec["name"], "host_bands": nb, "async": asyn, "ms_median": round(res[2], 3),
                          "mpix_s": round(W * H / res[2] / 1e3, 1)}), flush=True)

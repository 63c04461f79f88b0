"""The multi-pass merge launch (BCF_MULTI=1) under compute-sanitizer."""
import os
import sys

os.environ["BCF_MULTI"] = "1"
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_spaa_berneys25_b200 as bcf  # noqa: E402
import synthetic_inputs as si  # noqa: E402

x = si.uniform_u32(200003, 5)
t = torch.from_numpy(x.view(np.int32).copy()).cuda()
assert np.array_equal(bcf.sort(t).cpu().numpy().view(np.uint32), oracle.sort_u32(x))
print("sanitize_multi ok")

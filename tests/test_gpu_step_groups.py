"""Step groups (several local steps per CUDA-graph replay, ASGD_STEP_GROUP) run the same
kernels in the same order as one graph per step: the parameters and every per-step loss
after two mega-batches (a ragged last ticket included) are bitwise equal."""
import os
import subprocess
import sys

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


def _run(tmp_path, group, name, prec):
    out = str(tmp_path / f"g{group}_{name}_{prec}.npz")
    env = dict(os.environ, ASGD_STEP_GROUP=str(group))
    subprocess.run([sys.executable, os.path.join(HERE, "step_group_run.py"), out, name, prec], env=env,
                   check=True, timeout=600)
    return np.load(out)


@pytest.mark.parametrize("name,prec", [("eurlex4k", "bf16"), ("tiny", "fp32")])
def test_step_groups_bitwise_equal(tmp_path, name, prec):
    a = _run(tmp_path, 1, name, prec)
    for g in (4, 7):
        b = _run(tmp_path, g, name, prec)
        assert int(a["n"]) == int(b["n"]) == 24 and int(a["u"]) == int(b["u"])
        np.testing.assert_array_equal(a["losses"], b["losses"])
        np.testing.assert_array_equal(a["params"], b["params"])

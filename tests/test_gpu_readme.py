"""The README's Python usage example runs as written (GPU) and leaves a finite state."""
import os
import re

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_readme_python_example_runs():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.fail("GPU test run without a CUDA device")
    txt = open(os.path.join(ROOT, "README.md")).read()
    code = re.findall(r"```python\n(.*?)```", txt, re.S)
    assert code, "no python block in README"
    ns = {}
    exec(compile(code[0], "README.md", "exec"), ns)
    S, F = ns["S"], ns["F"]
    assert S.check_state() == 0 and F.check_state() == 0
    S.close()
    F.close()

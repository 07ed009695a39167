import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)
HERE = os.path.dirname(os.path.abspath(__file__))
if HERE not in sys.path:
    sys.path.insert(0, HERE)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running")


# ---------------------------------------------------------------------------
# Path coverage of the GPU suite: after every GPU test the engines it created
# (tests/gpu_helpers.make_pair) report which code paths answered its work
# (DUM_CTR_Q_*, DUM_CTR_WALK_*, ...); the totals are written at session end
# to gpurun_out/path_counters.json (or $DUM_PATHS_OUT) and checked by
# test_gpu_zz_paths.py::test_every_path_taken_in_the_suite (runs last).
# ---------------------------------------------------------------------------
import collections  # noqa: E402
import json  # noqa: E402

import pytest  # noqa: E402

PATHS = ["Q_FAST", "Q_NODUP", "Q_DUP", "Q_FALLBACK", "WALK_PREFIX", "WALK_DEDUPE", "WALK_SLOW", "ANCHOR_WALKS",
         "INGEST_DUP", "Q_SLOW", "FAST_DIRTY"]
PATH_TOTALS = collections.Counter()
PATH_BY_TEST = {}


@pytest.fixture(autouse=True)
def _collect_path_counters(request):
    yield
    if request.node.get_closest_marker("gpu") is None:
        return
    try:
        import gpu_helpers
    except Exception:
        return
    got = collections.Counter()
    for eng in gpu_helpers.LIVE_ENGINES:
        try:
            c = eng.counters()
        except Exception:
            continue
        for k in PATHS:
            got[k] += c.get(k, 0)
    gpu_helpers.LIVE_ENGINES.clear()
    PATH_TOTALS.update(got)
    PATH_BY_TEST[request.node.nodeid] = {k: v for k, v in got.items() if v}


def pytest_sessionfinish(session, exitstatus):
    if not PATH_BY_TEST:
        return
    out = os.environ.get("DUM_PATHS_OUT") or os.path.join(ROOT, "gpurun_out", "path_counters.json")
    try:
        os.makedirs(os.path.dirname(out), exist_ok=True)
        with open(out, "w") as fh:
            json.dump({"totals": dict(PATH_TOTALS), "by_test": PATH_BY_TEST}, fh, indent=1)
    except OSError:
        pass

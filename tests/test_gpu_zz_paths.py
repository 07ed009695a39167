"""Path coverage of the GPU suite (runs last: file order).  Every code path
that answers the engine's work must have answered some of the suite's:
  Q_FAST / Q_SLOW        fast windows (k_window_fast: pairs + selection; k_copy_fast without selection)
                         and the exact kernel (k_predict)
  Q_NODUP / Q_DUP / Q_FALLBACK  the exact kernel's window-set, duplicate and
                         fallback paths
  WALK_PREFIX / WALK_DEDUPE / WALK_SLOW  the three walk builders
  ANCHOR_WALKS           fault-anchored queries (D14)
  INGEST_DUP             launches with repeated blocks at ingest
  FAST_DIRTY             the fast selection on a log with stale entries
The counters come from tests/conftest.py (read from every engine a test
created); a partial run (-k) is not judged."""
from __future__ import annotations

import pytest
import torch

import conftest

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)


def test_every_path_taken_in_the_suite(request):
    n_gpu = sum(1 for it in request.session.items if it.get_closest_marker("gpu") is not None)
    if len(conftest.PATH_BY_TEST) < n_gpu - 1 or n_gpu < 100:
        pytest.skip("partial GPU run (%d of %d tests): coverage not judged" % (len(conftest.PATH_BY_TEST), n_gpu))
    missing = [k for k in conftest.PATHS if conftest.PATH_TOTALS.get(k, 0) == 0]
    assert not missing, "paths never taken by the GPU suite: %s (totals %s)" % (missing, dict(conftest.PATH_TOTALS))

"""GPU parity of every ablation knob setting (DESIGN.md's ablation table) (-m gpu).

The knobs select compiled kernel variants (pass configurations, table sizes, key formats,
vertex numbering) that the default path never launches; the ablation numbers in DESIGN.md
are only meaningful if those variants are exact too. Each setting runs tests/knob_parity.py
in a fresh process (the library reads the environment once) and must match the oracle bit
for bit on scaled BASELINE configs.
"""
import os
import subprocess
import sys

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

HERE = os.path.dirname(os.path.abspath(__file__))

KNOBS = [
    {"MST_PASSCFG": "1"},        # <24,4,2>
    {"MST_PASSCFG": "2"},        # <16,8,2>: 256 arcs per consumer warp
    {"MST_PASSCFG": "3"},        # <24,4,3>: 3-stage ring
    {"MST_PASSCFG": "4"},        # <30,4,3>
    {"MST_MIN0_CFG": "2"},       # the round-0 pass in its own configuration
    {"MST_QFILTER": "0"},        # no quantised-weight filter
    {"MST_QFILTER": "2"},        # filter tables in every filter pass
    {"MST_REORDER": "0"},        # caller's vertex numbering (no hub-first layout)
    {"MST_REORDER": "2"},        # BFS-order layout (NEXT-4)
    {"MST_PACKED_KEYS": "0"},    # always (w << 32) | eid keys
    {"MST_OWNER_MAX": "0"},      # lower internal id owns each record
    {"MST_HUB_ROW": "0"},
    {"MST_HUB_ROW": "1"},
    {"MST_MIN0_HOT": "0"},       # no shared hot-prefix table in the round-0 pass
    {"MST_MIN0_HOT": "1000"},
    {"MST_FILTER_HOT": "0"},
    {"MST_LIGHT_SWITCH": "2"},
    {"MST_LIGHT_T": "3"},        # forced light threshold (deferred vertices, extra passes)
    {"MST_LIGHT_K": "1"},
    {"MST_LIGHT_ONLY0": "1"},
    {"MST_LIGHT_ONLY0": "0"},
    {"MST_MEMBER_SCAN": "0"},    # always a pass over every record after the light phase
    {"MST_LIGHT_COMPACT": "1"},  # light-phase passes compact (adaptive) from round 1
    {"MST_LIGHT_COMPACT": "2"},  # ... always from round 1 (member decisions on compacted records)
    {"MST_LIGHT_COMPACT": "3"},  # ... adaptive from round 0
    {"MST_LIGHT_COMPACT": "2", "MST_LIGHT_T": "3"},
    {"MST_TX_DEDUP": "0"},       # dense transition: no warp merge of equal cells
    {"MST_TX_DEDUP": "1"},       # ... also without a hub row
    {"MST_ADJ_DEDUP": "0"},      # no adjacent-duplicate filter in compacting passes
    {"MST_ADJ_DEDUP": "1"},      # ... on everywhere (also BFS-ordered graphs)
    {"MST_REORDER": "1"},        # hub-first even where the auto rule picks BFS order
    {"MST_SMALL": "0"},          # no one-CTA path (grid64 through the multi-kernel path)
    {"MST_TEST_OPTIONS": "6=1"},                     # union-find variant (NEXT-3)
    {"MST_TEST_OPTIONS": "6=1", "MST_UF_TAG": "0"},  # ... untagged keys, best reset per round
    {"MST_TEST_OPTIONS": "6=1,4=1000"},              # ... always compacting
]


@pytest.mark.parametrize("env", KNOBS, ids=lambda e: ",".join(f"{k}={v}" for k, v in e.items()))
def test_knob_parity(env):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    full = dict(os.environ)
    full.update(env)
    r = subprocess.run([sys.executable, os.path.join(HERE, "knob_parity.py")], env=full,
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, (env, r.stdout[-2000:], r.stderr[-4000:])
    assert r.stdout.strip().splitlines()[-1].startswith("ok "), r.stdout[-2000:]

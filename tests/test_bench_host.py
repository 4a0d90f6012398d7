"""bench.py host logic that needs no GPU: the helper-process JSON collection of the secondary legs."""
import sys

import bench


def test_json_lines_collects_objects_and_errors():
    code = "import json; print('noise'); print(json.dumps({'a': 1})); print(json.dumps({'b': 2}))"
    assert bench._json_lines([sys.executable, "-c", code], {}, 60) == [{"a": 1}, {"b": 2}]
    bad = bench._json_lines([sys.executable, "-c", "import sys; sys.stderr.write('boom\\n'); sys.exit(3)"], {}, 60)
    assert len(bad) == 1 and "rc=3" in bad[0]["error"] and "boom" in bad[0]["error"]
    slow = bench._json_lines([sys.executable, "-c", "import time; time.sleep(5)"], {}, 0.5)
    assert slow == [{"error": "timeout after 0s"}] or "timeout" in slow[0]["error"]

"""Instrumented-kernel slowdowns (bench.measure_slowdown) on their own."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402

print(json.dumps(bench.measure_slowdown(0), indent=1))

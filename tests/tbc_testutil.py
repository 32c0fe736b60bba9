"""Shared helpers for the test-suite (no method arithmetic)."""
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def golden(name):
    """Load a fixture from tests/golden/ (each one states its citation)."""
    with open(os.path.join(ROOT, "tests", "golden", name)) as f:
        return json.load(f)

"""Test helpers shared by tests/ (file locations, golden-file parsing)."""
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def golden_path(name: str) -> str:
    return os.path.join(ROOT, "tests", "golden", name)


def golden_rows(name: str):
    rows = []
    with open(golden_path(name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows

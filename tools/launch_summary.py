"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV) per kernel: python tools/launch_summary.py x.csv"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from profile_collect import launch_summary  # noqa: E402

if __name__ == "__main__":
    launch_summary(sys.argv[1], "/dev/stdout")

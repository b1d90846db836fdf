timeout 1500 python -m pytest tests -q -x -m gpu 2>&1 | tail -3
python tools/convert_probe.py

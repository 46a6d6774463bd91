timeout 300 python tools/dec_time.py mix text zeroruns random 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -1

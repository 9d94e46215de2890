for o in 1e4 1e6; do timeout 120 python tools/ingest_probe.py $o 1e7 5; done 2>&1
timeout 120 python tools/ingest_probe.py 1e6 1e8 3 2>&1
timeout 120 python tools/ingest_probe.py 1e6 6.4e7 3 C3 2>&1
timeout 400 python -m pytest tests -m gpu -x -q 2>&1 | tail -2

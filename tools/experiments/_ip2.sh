for m in 0 3; do for b in 10000 1000000; do
GG_INGEST_KERNELS=$m ncu --metrics gpu__time_duration.sum,smsp__cycles_active.avg --clock-control none --csv -k regex:k_ingest python tools/ingest_probe.py 10000 $b 3 2>/dev/null | grep -E "k_ingest" | awk -F'","' '{print "'m$m' b'$b'", $5, $(NF-2), $NF}' | tail -4
done; done

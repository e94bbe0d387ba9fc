# merged CTA votes: parity; phase profile; C5 group times; source-level ncu of one heavy 64-GPU C5 point (prof build)
O=gpurun_out/s4k
mkdir -p $O
timeout 1800 python -m pytest tests -m gpu -q -x > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
TRIOSIM_LIB=paper_conf_isca_libwmvgjbj025_b200/libtriosim_prof.so timeout 600 python tools/c5_prof.py 64 512 1024 > $O/c5prof.log 2>&1
timeout 900 python tools/c5_subset.py 64 128 256 > $O/c5sub.log 2>&1; echo "rc=$?" >> $O/c5sub.log
TRIOSIM_LIB=paper_conf_isca_libwmvgjbj025_b200/libtriosim_prof.so timeout 900 ncu -f --set full --clock-control none --import-source on -k regex:k3_hybrid -o /tmp/c5pt python tools/c5_points.py 28 > $O/ncu_c5pt.log 2>&1
ncu -i /tmp/c5pt.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > $O/src_c5pt.csv.gz
ncu -i /tmp/c5pt.ncu-rep --page raw --csv > $O/raw_c5pt.csv 2>&1
ls -la $O

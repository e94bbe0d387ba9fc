# CTA water-filling with fire-and-forget counts and per-link passes: parity (incl. the C5 goldens up to 256 GPUs),
# phase profile, C5 group times per N (new vs previous build)
O=gpurun_out/s4j
mkdir -p $O
timeout 1800 python -m pytest tests -m gpu -q -x --durations=8 > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
TRIOSIM_LIB=paper_conf_isca_libwmvgjbj025_b200/libtriosim_prof.so timeout 600 python tools/c5_prof.py 64 512 1024 > $O/c5prof.log 2>&1
timeout 900 python tools/c5_subset.py 64 128 256 > $O/c5sub.log 2>&1; echo "rc=$?" >> $O/c5sub.log
TRIOSIM_LIB=paper_conf_isca_libwmvgjbj025_b200/libtriosim_prev.so timeout 300 python tools/c5_subset.py 64 > $O/c5sub_prev.log 2>&1
ls -la $O

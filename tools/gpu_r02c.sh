timeout 900 python -m pytest tests/test_gpu_stream.py -m gpu -q -x -p no:cacheprovider > gpurun_out/r02c_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02c_pytest.log
bash tools/gpu_variants.sh r02c pubmed hint1_z1 hint0_z1 hint1_z0 hint0_z0
tail -3 gpurun_out/r02c_pytest.log
bash tools/gpu_variants.sh r02c2 pubmed h1z0pf h0z0pf

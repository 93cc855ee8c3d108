# a x 1 row blocks: 20-epoch RMSE curves on the full Netflix shape + fullsize tests
python tools/fullsize_rmse.py > gpurun_out/r02ae_rmse.log 2>&1
python -m pytest tests/test_gpu_fullsize.py -q -p no:cacheprovider -k "variants" > gpurun_out/r02ae_tests.log 2>&1
tail -3 gpurun_out/r02ae_tests.log; grep "epoch 20" gpurun_out/r02ae_rmse.log

set -u
mkdir -p gpurun_out
bash tools/ncu_one.sh "k_csr_vector|k_csr_flat" C3 c3new
bash tools/ncu_one.sh "k_csr_vector|k_csr_flat" S3 s3new

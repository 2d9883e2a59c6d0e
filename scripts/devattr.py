"""dev: print the L2 / persisting-window device attributes of cuda:0."""
import cuda.bindings.runtime as r
for a in ("cudaDevAttrL2CacheSize", "cudaDevAttrMaxAccessPolicyWindowSize",
          "cudaDevAttrMaxPersistingL2CacheSize", "cudaDevAttrMultiProcessorCount"):
    err, v = r.cudaDeviceGetAttribute(getattr(r.cudaDeviceAttr, a), 0)
    print(a, v, err)
err, v = r.cudaDeviceGetLimit(r.cudaLimit.cudaLimitMaxL2FetchGranularity)
print("cudaLimitMaxL2FetchGranularity", v, err)

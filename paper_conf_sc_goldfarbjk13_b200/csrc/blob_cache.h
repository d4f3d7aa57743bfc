// blob_cache.h -- recycling of the device blobs of GPU-built trees.
#pragma once
#include <cstddef>

// Device blobs of GPU-built trees: cudaMalloc'd, recycled on tt_tree_free
// (after a device synchronisation) into a small cache (tt_api.cu).
int tt_blob_take(size_t bytes, void **out);  // a cudaError_t
void tt_blob_release(void *blob);  // caller guarantees the blob is idle (and on the current device)
void tt_blob_discard(void *blob);  // cudaFree, forgetting it (error paths, device not idle)
bool tt_blob_is_cached_kind(void *blob);
